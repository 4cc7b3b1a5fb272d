set -x
python tools/profile_query.py --part 0 --query K5-K2 --reps 2 --stats > gpurun_out/pq.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_extend -c 1 -o gpurun_out/r01_extend_K5K2 python tools/profile_query.py --part 0 --query K5-K2 > gpurun_out/ncu_full.log 2>&1
timeout 1200 python bench.py --steps 2 --warmup 3 > gpurun_out/bench_r01a.json 2> gpurun_out/bench_r01a.err
tail -3 gpurun_out/bench_r01a.err
cat gpurun_out/bench_r01a.json
