nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_g.log 2>&1; tail -15 gpurun_out/pytest_gpu_g.log
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout -k 10 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_r01g.json 2> gpurun_out/bench_r01g.err
cat gpurun_out/bench_r01g.json; tail -3 gpurun_out/bench_r01g.err
timeout -k 10 900 python tools/calibrate.py --scale 20 --ef 10 --abc 0.50,0.20,0.20 --abc 0.52,0.20,0.20 --abc 0.55,0.19,0.19 --family 6,7,8 --min-nparts 64 --budget 60 --out gpurun_out/calib_c3.jsonl > gpurun_out/calib_c3.log 2>&1
tail -2 gpurun_out/calib_c3.log
timeout -k 10 900 python tools/calibrate.py --scale 22 --ef 16 --abc 0.45,0.22,0.22 --abc 0.50,0.20,0.20 --abc 0.55,0.19,0.19 --family 8 --min-nparts 4096 --budget 600 --out gpurun_out/calib_c4.jsonl > gpurun_out/calib_c4.log 2>&1
tail -2 gpurun_out/calib_c4.log
