# HEAD re-check after container restore: build, full GPU suite, smoke, bench line, launch list
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build_s.log 2>&1 || tail -20 gpurun_out/build_s.log
timeout -k 10 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_s.log 2>&1; tail -3 gpurun_out/pytest_s.log
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_s.log 2>&1; tail -1 gpurun_out/smoke_s.log
timeout -k 10 600 python bench.py > gpurun_out/bench_s.json 2> gpurun_out/bench_s.err; tail -c 600 gpurun_out/bench_s.json
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_s.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/bench_s_ncu.log 2>&1; wc -l gpurun_out/launches_s.csv
