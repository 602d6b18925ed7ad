cd $GRAFT_REPO_ROOT
for v in default tb_shf tb_r96 tb_shf_r96 tb_g3; do
  lib=$PWD/exp/$v/libmapsm.so; [ $v = default ] && lib=$PWD/paper_conf_sc_ben_nunlbr15_b200/libmapsm.so
  for a in "life64k 48 --deep 4" "life64k 48 --deep 8" "life8k 48 --deep 8" "life8k 48 --deep 4"; do
    MAPSM_LIB=$lib timeout 120 python tools/kbench.py $a 2>&1 | tail -1 | python -c "
import sys,json
l=sys.stdin.read()
try:
  d=json.loads(l); print('$v', d['workload'], d['deep'], round(d['ms_per_launch']*1000,1), 'us/gen', round(d['cells_per_s']/1e12,2), 'T')
except Exception: print('$v', l[:300])"
  done
done
