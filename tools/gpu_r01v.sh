# launch-bound fix: bench line + launch list + C2 ablation (packed, reuse, full) + fast/first-source tests
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build_v.log 2>&1 || tail -20 gpurun_out/build_v.log
timeout -k 10 600 python bench.py > gpurun_out/bench_v.json 2> gpurun_out/bench_v.err; tail -c 300 gpurun_out/bench_v.json
timeout -k 10 600 python tools/ablation.py --workload C2 --reps 2 --variants packed,reuse,full --out gpurun_out/ablation_c2_v.jsonl > gpurun_out/ablation_v.log 2>&1; grep total_s gpurun_out/ablation_v.log
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/bench_v_ncu.log 2>&1; wc -l gpurun_out/launches_v.csv
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_v.log 2>&1; tail -1 gpurun_out/smoke_v.log
