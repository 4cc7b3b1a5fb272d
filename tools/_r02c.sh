python __graft_entry__.py > gpurun_out/r02c_build.log 2>&1
timeout -k 5 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c_launches.csv \
  python tools/c4_sweep.py --ranges pos:13997:13998 > gpurun_out/r02c_ncu_launch.log 2>&1; tail -2 gpurun_out/r02c_ncu_launch.log
timeout -k 5 900 ncu --set full --clock-control none --import-source on -k "regex:k_extend<7" -s 400 -c 1 -o gpurun_out/r02c_ext7 -f \
  python tools/c4_sweep.py --ranges pos:13997:13998 > gpurun_out/r02c_ncu7.log 2>&1; tail -2 gpurun_out/r02c_ncu7.log
timeout -k 5 900 ncu --set full --clock-control none --import-source on -k "regex:k_extend<6" -s 200 -c 2 -o gpurun_out/r02c_ext6 -f \
  python tools/c4_sweep.py --ranges pos:13997:13998 > gpurun_out/r02c_ncu6.log 2>&1; tail -2 gpurun_out/r02c_ncu6.log
timeout -k 5 900 ncu --set full --clock-control none --import-source on -k "regex:k_plan" -s 600 -c 1 -o gpurun_out/r02c_plan -f \
  python tools/c4_sweep.py --ranges pos:13997:13998 > gpurun_out/r02c_ncup.log 2>&1; tail -2 gpurun_out/r02c_ncup.log
timeout -k 5 1200 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=15 -k "next2 or dist or carry or disconnected_fullsize or fast_last or first_source or c4_root" > gpurun_out/r02c_pytest.log 2>&1; tail -25 gpurun_out/r02c_pytest.log
