nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu_f.log
cat gpurun_out/pytest_gpu_f.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r01f.json 2> gpurun_out/bench_r01f.err
cat gpurun_out/bench_r01f.json; tail -3 gpurun_out/bench_r01f.err
