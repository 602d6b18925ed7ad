cd $GRAFT_REPO_ROOT
for rep in 1 2; do bash tools/gpu_tune.sh conv9 c9_e2 c9_e2_2cta c9_e4 c9_e2_nc16; done 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    n,_,j=l.partition(' ')
    try: d=json.loads(j); print(n, round(d['ms_per_launch']*1000,1),'us', round(d['cells_per_s']/1e9),'Gcell/s')
    except Exception: print(l.strip()[:300])
"
