cd $GRAFT_REPO_ROOT
for wl in life64k conv5 conv9; do bash tools/gpu_tune.sh $wl pre_p2p pl1 pl2; done 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    n,_,j=l.partition(' ')
    try: d=json.loads(j); print(n, d['workload'], round(d['ms_per_launch']*1000,1),'us', round(d['GBps']),'GB/s')
    except Exception: print(l.strip()[:300])
"
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
