cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for v in pre_p2p cur; do
MAPSM_LIB=$PWD/exp/$v/libmapsm.so timeout 300 ncu --set full --clock-control none -k regex:life_tma -s 3 -c 1 -o gpurun_out/cmp_$v python tools/kbench.py life64k 4 > /dev/null 2>&1; echo $v=$?
done
