cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/pytest_gpu_r27.log 2>&1; echo pytest=$?; tail -n 3 gpurun_out/pytest_gpu_r27.log
timeout 600 python bench.py > gpurun_out/bench_default_r27.json 2>gpurun_out/bench_default_r27.err; echo bench=$?; cat gpurun_out/bench_default_r27.json
timeout 300 python bench.py --workload conv9 --steps 5 --warmup 3 > gpurun_out/bench_conv9_r27.json 2>>gpurun_out/v.err; echo conv9=$?; cat gpurun_out/bench_conv9_r27.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/conv9_launches_r27.csv python bench.py --workload conv9 --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/conv9_ncu_r27.log 2>&1; echo ncu=$?
timeout 120 python -c "import __graft_entry__ as g; g.smoke()"; echo smoke=$?
