cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
for wl in life64k conv5; do timeout 120 python tools/kbench.py $wl 20; done
for wl in life64k conv5; do for g in 2 4 8; do for x in copy p2p; do timeout 120 python tools/kbench.py $wl 20 --local $g --exchange $x; done; done; done
