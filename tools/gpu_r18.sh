cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_conv3d.py -x -q --timeout 600 > gpurun_out/pytest_conv3d.log 2>&1; echo pytest=$?; tail -30 gpurun_out/pytest_conv3d.log
timeout 600 python bench.py --workload conv3d --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_conv3d.json 2>> gpurun_out/bench.err; echo bench=$?; cat gpurun_out/bench_conv3d.json
tail -5 gpurun_out/bench.err
ncu --set full --import-source on -k regex:conv3d_kernel -s 20 -c 1 -o gpurun_out/conv3d_full python bench.py --workload conv3d --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_conv3d.log 2>&1; echo ncu=$?; tail -3 gpurun_out/ncu_conv3d.log
