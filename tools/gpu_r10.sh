cd $GRAFT_REPO_ROOT
for rep in 1 2; do bash tools/gpu_tune.sh life64k pre_p2p cur; bash tools/gpu_tune.sh conv5 pre_p2p cur; done 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    n,_,j=l.partition(' ')
    try: d=json.loads(j); print(n, d['workload'], round(d['ms_per_launch']*1000,1),'us', round(d['GBps']),'GB/s')
    except Exception: print(l.strip()[:300])
"
