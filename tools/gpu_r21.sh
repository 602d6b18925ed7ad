cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_conv3d.py -x -q --timeout 600 > gpurun_out/pytest_conv3d.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_conv3d.log
for w in conv3d conv3d5; do
timeout 300 python bench.py --workload $w --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_$w.json 2>>gpurun_out/v.err; echo $w $(python -c "import json;d=json.load(open('gpurun_out/bench_$w.json'));r=d['roofline'];print(d['value'], r['kernel_ms_per_launch'], r['frac'], r['fma_frac_at_sampled_clock'])")
done
ncu --set full --import-source on -k regex:conv3d_kernel -s 20 -c 1 -o gpurun_out/conv3d_full python bench.py --workload conv3d --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_conv3d.log 2>&1; echo ncu=$?
