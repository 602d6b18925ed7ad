cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ./exp/bin/membench | tee gpurun_out/membench.txt
