cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for rep in 1 2; do
bash tools/gpu_tune.sh life64k r6 t8_12 t8_12_c1 t8_12_c2 t16_12_c1 t16_6_c2 t8_24_c2 t16_24_c1 t24_9_c1
done > gpurun_out/tune4.txt 2>&1
cat gpurun_out/tune4.txt | python -c "
import sys,json
for l in sys.stdin:
    n,_,j=l.partition(' ')
    try: d=json.loads(j); print(n, round(d['ms_per_launch']*1000,1),'us', round(d['GBps']),'GB/s', round(d['region_GBps']))
    except Exception: print(l.strip()[:200])
"
