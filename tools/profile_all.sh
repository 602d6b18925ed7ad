#!/usr/bin/env bash
# tools/profile_all.sh TAG — ncu evidence for every timed kernel (run through gpurun):
#   ncu --set full of one launch of each dominant kernel + the launch list of the
#   default bench (headline only); reports land in gpurun_out/TAG_*.
cd "${GRAFT_REPO_ROOT:-$(pwd)}"
mkdir -p gpurun_out
T=$1
full() {  # name regex skip cmd...
  local name=$1 re=$2 skip=$3; shift 3
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$re -s $skip -c 1 \
    -o gpurun_out/${T}_$name "$@" > gpurun_out/${T}_$name.log 2>&1
  echo "$name rc=$?"
}
full life64k life_tma 8 python tools/kbench.py life64k 4
full life8k life_resident 4 python tools/rbench.py --reps 1
full conv5 conv_tma 8 python tools/kbench.py conv5 4
full conv9 conv_tma 8 python tools/kbench.py conv9 4
full life64k_tb8 life_tb 4 python tools/kbench.py life64k 4 --deep 8
full hist8k histogram 3 python bench.py --workload hist8k --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
  --log-file gpurun_out/${T}_life64k_bench_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline \
  --e2e-steps 1 --no-configs --deep-halo 0 > gpurun_out/${T}_launches.log 2>&1
echo "launches rc=$?"
