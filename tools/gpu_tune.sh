# usage: bash tools/gpu_tune.sh <workload> <variant dirs...>
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
wl=$1; shift
for v in "$@"; do
  MAPSM_LIB=$PWD/exp/$v/libmapsm.so timeout 120 python tools/kbench.py $wl 20 2>&1 | tail -1 | sed "s/^/$v /"
done
