#!/usr/bin/env bash
# tools/gpu.sh — the one GPU-box runner (invoked through gpurun):
#   gpurun --timeout 1800 -- 'bash tools/gpu.sh TAG STEP [STEP ...]'
# Every output lands in gpurun_out/TAG_*.  Steps:
#   smoke                 __graft_entry__.smoke()
#   tests[=EXPR]          pytest -m gpu [-k EXPR]
#   bench[=ARGS]          python bench.py ARGS (default: the driver's default run)
#   launches[=ARGS]       ncu launch list (gpu__time_duration) of bench.py ARGS
#   ncu=REGEX[:ARGS]      ncu --set full of the first launch of kernels matching
#                         REGEX while running `python ARGS` (e.g.
#                         ncu=conv_tma:tools/kbench.py,conv9,4 or
#                         ncu=life_resident:bench.py,--workload,life8k,--steps,1)
#   sanitize              compute-sanitizer memcheck/racecheck/synccheck of tools/sanitize_cases.py
# ARGS use ',' for spaces (e.g. bench=--workload,conv9,--steps,5).
set -u
cd "${GRAFT_REPO_ROOT:-$(pwd)}"
mkdir -p gpurun_out
TAG=$1
shift
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv,noheader > gpurun_out/${TAG}_gpu.txt
nproc >> gpurun_out/${TAG}_gpu.txt
for step in "$@"; do
  name=${step%%=*}
  arg=""
  [[ "$step" == *=* ]] && arg=${step#*=}
  arg=${arg//,/ }
  case $name in
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
      echo "smoke rc=$?"; tail -2 gpurun_out/${TAG}_smoke.log ;;
    tests)
      n=$(ls gpurun_out/${TAG}_pytest*.log 2>/dev/null | wc -l)
      if [ -n "$arg" ]; then
        timeout 3000 python -m pytest tests -m gpu -q --timeout 1200 -k "$arg" > gpurun_out/${TAG}_pytest$n.log 2>&1
      else
        timeout 3000 python -m pytest tests -m gpu -q --timeout 1200 > gpurun_out/${TAG}_pytest$n.log 2>&1
      fi
      echo "pytest$n rc=$?"; tail -4 gpurun_out/${TAG}_pytest$n.log ;;
    bench)
      n=$(ls gpurun_out/${TAG}_bench*.json 2>/dev/null | wc -l)
      timeout 900 python bench.py $arg > gpurun_out/${TAG}_bench$n.json 2> gpurun_out/${TAG}_bench$n.err
      echo "bench$n rc=$?"; cat gpurun_out/${TAG}_bench$n.json; tail -3 gpurun_out/${TAG}_bench$n.err ;;
    launches)
      [ -z "$arg" ] && arg="--steps 2 --warmup 1"
      timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
        --log-file gpurun_out/${TAG}_launches.csv python bench.py $arg > gpurun_out/${TAG}_launches.log 2>&1
      echo "launches rc=$?" ;;
    ncu)
      re=${arg%%:*}; ka=""; [[ "$arg" == *:* ]] && ka=${arg#*:}
      n=$(ls gpurun_out/${TAG}_ncu*.ncu-rep 2>/dev/null | wc -l)
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:$re -s ${NCU_SKIP:-2} -c 1 \
        -o gpurun_out/${TAG}_ncu$n python $ka > gpurun_out/${TAG}_ncu$n.log 2>&1
      echo "ncu$n rc=$?"
      ncu -i gpurun_out/${TAG}_ncu$n.ncu-rep --page raw --csv > gpurun_out/${TAG}_ncu$n.raw.csv 2>/dev/null ;;
    sanitize)
      for tool in memcheck racecheck synccheck; do
        timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_cases.py \
          > gpurun_out/${TAG}_sanitize_$tool.log 2>&1
        echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|ALL OK|FAILURES|MISMATCH" \
          gpurun_out/${TAG}_sanitize_$tool.log | tail -3
      done ;;
    *) echo "unknown step $name" ;;
  esac
done
