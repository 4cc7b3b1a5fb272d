nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 600 python -m pytest tests/test_gpu_fullsize.py -x -q > gpurun_out/pytest_fullsize_i.log 2>&1; tail -5 gpurun_out/pytest_fullsize_i.log
timeout -k 10 900 python tools/calibrate.py --scale 20 --ef 10 --abc 0.50,0.20,0.20 --abc 0.52,0.20,0.20 --abc 0.55,0.19,0.19 --family 6,7,8 --min-nparts 64 --budget 60 --out gpurun_out/calib_c3.jsonl > gpurun_out/calib_c3.log 2>&1
tail -2 gpurun_out/calib_c3.log
timeout -k 10 1200 python tools/calibrate.py --scale 22 --ef 16 --abc 0.45,0.22,0.22 --abc 0.50,0.20,0.20 --abc 0.55,0.19,0.19 --family 8 --min-nparts 4096 --budget 600 --out gpurun_out/calib_c4.jsonl > gpurun_out/calib_c4.log 2>&1
tail -2 gpurun_out/calib_c4.log
