python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_donation.py -x -q 2>&1 | tail -2
timeout -k 10 300 python tools/sweep.py --workload C2 --hub 0 --reps 2 --out gpurun_out/sweep_c2_o.jsonl > gpurun_out/sweep_c2_o.log 2>&1; grep total_s gpurun_out/sweep_c2_o.log
