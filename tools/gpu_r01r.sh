nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_donation.py -x -q > gpurun_out/pytest_r.log 2>&1; tail -3 gpurun_out/pytest_r.log
timeout -k 10 300 python tools/sweep.py --workload C2 --hub 0 --reps 2 --out gpurun_out/sweep_c2_r.jsonl > gpurun_out/sweep_c2_r.log 2>&1; grep total_s gpurun_out/sweep_c2_r.log
timeout -k 10 300 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_extend<\(int\)4, \(int\)1, \(int\)1' -s 5 -c 1 -o gpurun_out/r01r_extend_last_K5C4 python tools/profile_query.py --part 0 --query K5-C4 > gpurun_out/ncu_k5c4_r.log 2>&1; tail -1 gpurun_out/ncu_k5c4_r.log
