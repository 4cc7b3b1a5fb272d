nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_l.log 2>&1; tail -3 gpurun_out/pytest_l.log
timeout -k 10 300 python tools/sweep.py --workload C2 --hub 0 --reps 2 --out gpurun_out/sweep_c2_l.jsonl > gpurun_out/sweep_c2_l.log 2>&1; grep total_s gpurun_out/sweep_c2_l.log
