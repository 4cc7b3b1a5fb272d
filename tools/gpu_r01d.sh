timeout 300 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_extend<\(int\)4, \(int\)1' -s 5 -c 1 -o gpurun_out/r01_extend_last_K5C4 python tools/profile_query.py --part 0 --query K5-C4 > gpurun_out/ncu_k5c4.log 2>&1
tail -2 gpurun_out/ncu_k5c4.log
