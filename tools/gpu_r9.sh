cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_p2p.py -x -q > gpurun_out/pytest_p2p.log 2>&1; echo p2p=$?; tail -15 gpurun_out/pytest_p2p.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for wl in life64k conv5; do timeout 120 python tools/kbench.py $wl 20; done
