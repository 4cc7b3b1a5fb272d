nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 900 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r01p.json 2> gpurun_out/bench_r01p.err
cat gpurun_out/bench_r01p.json; tail -3 gpurun_out/bench_r01p.err
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv --log-file gpurun_out/r01p_launches_bench.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_bench_p.log 2>&1; tail -1 gpurun_out/ncu_bench_p.log
timeout -k 10 300 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_extend<\(int\)4, \(int\)1, \(int\)1' -s 5 -c 1 -o gpurun_out/r01p_extend_last_K5C4 python tools/profile_query.py --part 0 --query K5-C4 > gpurun_out/ncu_k5c4_p.log 2>&1; tail -1 gpurun_out/ncu_k5c4_p.log
timeout -k 10 2400 python tools/c4_run.py --out gpurun_out/c4_run_p.json > gpurun_out/c4_run_p.log 2>&1; tail -3 gpurun_out/c4_run_p.log
