nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_h.log 2>&1; tail -15 gpurun_out/pytest_gpu_h.log
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout -k 10 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r01h.json 2> gpurun_out/bench_r01h.err
cat gpurun_out/bench_r01h.json; tail -3 gpurun_out/bench_r01h.err
