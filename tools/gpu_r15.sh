cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_life64k.json 2> gpurun_out/bench.err; echo bench=$?; cat gpurun_out/bench_life64k.json; tail -3 gpurun_out/bench.err
timeout 600 python bench.py --workload life8k --steps 5 --warmup 3 > gpurun_out/bench_life8k.json 2>> gpurun_out/bench.err; echo bench8k=$?; cat gpurun_out/bench_life8k.json
