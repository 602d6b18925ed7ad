cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_deep_halo.py -x -q > gpurun_out/pytest_tb.log 2>&1; echo pytest_tb=$?; tail -3 gpurun_out/pytest_tb.log
for a in "life64k 48 --deep 4" "life64k 48 --deep 6" "life64k 48 --deep 8" "life8k 48 --deep 4" "life8k 48 --deep 6" "life8k 48 --deep 8"; do
  timeout 120 python tools/kbench.py $a 2>&1 | tail -1 | python -c "
import sys,json
l=sys.stdin.read()
try:
  d=json.loads(l); print(d['workload'], d['deep'], round(d['ms_per_launch']*1000,1), 'us/gen', round(d['cells_per_s']/1e12,2), 'T')
except Exception: print(l[:300])"
done
