cd $GRAFT_REPO_ROOT
for v in $(ls exp); do
  MAPSM_LIB=exp/$v/libmapsm.so timeout 300 python tools/rbench.py 2>&1 | tail -1
done
