cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for wl in hist8k life64k; do timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 > gpurun_out/bench_$wl.json 2> gpurun_out/bench_$wl.err; echo $wl=$?; cat gpurun_out/bench_$wl.json; tail -2 gpurun_out/bench_$wl.err; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:histogram_kernel -s 3 -c 1 -o gpurun_out/prof_hist python bench.py --workload hist8k --steps 2 --warmup 1 --e2e-steps 1 --no-cpu-baseline > gpurun_out/ncu_hist.log 2>&1; echo ncu=$?
