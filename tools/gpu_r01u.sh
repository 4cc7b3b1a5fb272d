# fast last-level count: new tests, bench line, launch list, ablation (reuse vs full), whole suite
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build_u.log 2>&1 || tail -20 gpurun_out/build_u.log
timeout -k 10 900 python -m pytest tests/test_gpu_parity.py -k "fast_last or first_source" -x -q > gpurun_out/pytest_u_new.log 2>&1; tail -15 gpurun_out/pytest_u_new.log
timeout -k 10 600 python bench.py > gpurun_out/bench_u.json 2> gpurun_out/bench_u.err; tail -c 400 gpurun_out/bench_u.json
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_u.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/bench_u_ncu.log 2>&1; wc -l gpurun_out/launches_u.csv
timeout -k 10 600 python tools/ablation.py --workload C2 --reps 2 --variants reuse,full --out gpurun_out/ablation_c2_u.jsonl > gpurun_out/ablation_u.log 2>&1; grep total_s gpurun_out/ablation_u.log
timeout -k 10 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_u.log 2>&1; tail -5 gpurun_out/pytest_u.log
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_u.log 2>&1; tail -1 gpurun_out/smoke_u.log
