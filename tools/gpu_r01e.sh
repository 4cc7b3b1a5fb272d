nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r01b.json 2> gpurun_out/bench_r01b.err
cat gpurun_out/bench_r01b.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 12000 --csv --log-file gpurun_out/r01_launches_bench.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
tail -2 gpurun_out/ncu_bench.log
