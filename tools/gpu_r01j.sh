nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python __graft_entry__.py > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 600 python tools/sweep.py --workload C2 --hub 0,64,off --reps 2 --out gpurun_out/sweep_c2_j.jsonl > gpurun_out/sweep_c2_j.log 2>&1; grep total_s gpurun_out/sweep_c2_j.log
timeout -k 10 300 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_extend<\(int\)4, \(int\)1' -s 5 -c 1 -o gpurun_out/r01j_extend_last_K5C4 python tools/profile_query.py --part 0 --query K5-C4 > gpurun_out/ncu_k5c4_j.log 2>&1
tail -2 gpurun_out/ncu_k5c4_j.log
timeout -k 10 700 python tools/calibrate.py --scale 20 --ef 10 --abc 0.47,0.22,0.22 --abc 0.48,0.21,0.21 --family 6,7,8 --min-nparts 64 --budget 60 --out gpurun_out/calib_c3_j.jsonl > gpurun_out/calib_c3_j.log 2>&1
timeout -k 10 600 python tools/calibrate.py --scale 22 --ef 16 --abc 0.47,0.22,0.22 --abc 0.48,0.21,0.21 --family 8 --only K8,K8-C4 --min-nparts 4096 --budget 600 --out gpurun_out/calib_c4_j.jsonl > gpurun_out/calib_c4_j.log 2>&1
