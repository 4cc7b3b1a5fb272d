set -x
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_extend<\(int\)4, \(int\)1>' -c 1 -o gpurun_out/r01_extend_last_K5K2 python tools/profile_query.py --part 0 --query K5-K2 > gpurun_out/ncu_full2.log 2>&1
tail -3 gpurun_out/ncu_full2.log
