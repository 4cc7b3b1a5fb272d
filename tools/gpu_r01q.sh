nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_donation.py -x -q > gpurun_out/pytest_q.log 2>&1; tail -3 gpurun_out/pytest_q.log
timeout -k 10 300 python tools/sweep.py --workload C2 --hub 0 --reps 2 --out gpurun_out/sweep_c2_q.jsonl > gpurun_out/sweep_c2_q.log 2>&1; grep total_s gpurun_out/sweep_c2_q.log
timeout -k 10 1200 python tools/sweep.py --workload C3 --hub 0 --reps 1 --out gpurun_out/sweep_c3_q.jsonl > gpurun_out/sweep_c3_q.log 2>&1; grep total_s gpurun_out/sweep_c3_q.log; tail -2 gpurun_out/sweep_c3_q.log
timeout -k 10 1800 python tools/c4_run.py --skip-bfs --out gpurun_out/c4_run_q.json > gpurun_out/c4_run_q.log 2>&1; tail -2 gpurun_out/c4_run_q.log
