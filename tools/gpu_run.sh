#!/bin/bash
# One parameterised GPU job (run under gpurun from the repo root):
#   tools/gpu_run.sh TAG STEP [STEP ...]
# Steps: build | tests | smoke | bench[:ARGS] | c4sweep[:RANGES] | ncu_launch[:ARGS] | ncu_full[:REGEX:SKIP:ARGS] | sanitize
# Every step writes gpurun_out/TAG_<step>.* and is wrapped in its own timeout.
tag=$1; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.used --format=csv,noheader > gpurun_out/${tag}_smi.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/${tag}_smi.txt; nproc >> gpurun_out/${tag}_smi.txt
for st in "$@"; do
  name=${st%%:*}; arg=""; [[ "$st" == *:* ]] && arg=${st#*:}
  t0=$(date +%s)
  case $name in
    build) timeout -k 10 600 python __graft_entry__.py > gpurun_out/${tag}_build.log 2>&1 ;;
    tests) timeout -k 10 ${arg:-1500} python -m pytest tests -m gpu -q --durations=40 -p no:cacheprovider \
             > gpurun_out/${tag}_pytest.log 2>&1; tail -45 gpurun_out/${tag}_pytest.log ;;
    testk) timeout -k 10 1200 python -m pytest tests -m gpu -q --durations=20 -p no:cacheprovider -k "$arg" \
             > gpurun_out/${tag}_pytestk.log 2>&1; tail -25 gpurun_out/${tag}_pytestk.log ;;
    smoke) timeout -k 10 300 python __graft_entry__.py --smoke > gpurun_out/${tag}_smoke.log 2>&1; tail -3 gpurun_out/${tag}_smoke.log ;;
    bench) timeout -k 10 1800 python bench.py $arg > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
           tail -c 3000 gpurun_out/${tag}_bench.json; tail -5 gpurun_out/${tag}_bench.err ;;
    c4sweep) timeout -k 10 1500 python tools/c4_sweep.py --ranges ${arg//,/ } --out gpurun_out/${tag}_c4sweep.jsonl \
             > gpurun_out/${tag}_c4sweep.log 2>&1; tail -c 2500 gpurun_out/${tag}_c4sweep.log ;;
    script) timeout -k 10 1800 bash -c "$arg" > gpurun_out/${tag}_script.log 2>&1; tail -c 3000 gpurun_out/${tag}_script.log ;;
    ncu_launch) timeout -k 10 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
             --log-file gpurun_out/${tag}_launches.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline $arg \
             > gpurun_out/${tag}_ncu_launch.log 2>&1; tail -3 gpurun_out/${tag}_ncu_launch.log ;;
    ncu_full) IFS=: read -r rx skip rest <<< "$arg"
             timeout -k 10 1800 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:${rx}" -s ${skip:-0} -c 1 \
             -o gpurun_out/${tag}_full -f $rest > gpurun_out/${tag}_ncu_full.log 2>&1; tail -5 gpurun_out/${tag}_ncu_full.log ;;
    sanitize) for tool in ${arg:-memcheck racecheck synccheck}; do
               timeout -k 10 1200 compute-sanitizer --tool $tool --error-exitcode 9 \
                 python tools/sanitize_run.py > gpurun_out/${tag}_sanitize_${tool}.log 2>&1
               echo "sanitize $tool rc=$?"; tail -4 gpurun_out/${tag}_sanitize_${tool}.log; done ;;
    *) echo "unknown step $name" ;;
  esac
  echo "== $tag $st rc=$? $(( $(date +%s) - t0 )) s"
done
