# k_plan<J, directed> (undirected plans back to J list slots): bench line + ablation full + directed/fast tests
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build_w.log 2>&1 || tail -20 gpurun_out/build_w.log
timeout -k 10 400 python bench.py > gpurun_out/bench_w.json 2> gpurun_out/bench_w.err; tail -c 200 gpurun_out/bench_w.json
timeout -k 10 300 python tools/ablation.py --workload C2 --reps 2 --variants full --out gpurun_out/ablation_c2_w.jsonl > gpurun_out/ablation_w.log 2>&1; grep total_s gpurun_out/ablation_w.log
timeout -k 10 600 python -m pytest tests/test_gpu_directed.py tests/test_gpu_parity.py -k "directed or fast_last or c1_er1000 or disconnected_levels" -x -q > gpurun_out/pytest_w.log 2>&1; tail -3 gpurun_out/pytest_w.log
