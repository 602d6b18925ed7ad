cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_conv.py tests/test_gpu_p2p.py -x -q --timeout 600 > gpurun_out/pytest_conv_r23.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_conv_r23.log
for w in conv9 conv5; do
timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_${w}_r23.json 2>>gpurun_out/v.err; echo $w $(python -c "import json;d=json.load(open('gpurun_out/bench_${w}_r23.json'));r=d['roofline'];print(d['value'], r.get('kernel_ms_per_launch'), r['frac'], r.get('fma_frac_at_sampled_clock'), d['clocks'])")
done
ncu --set full --import-source on -k regex:conv_tma_kernel -s 6 -c 1 -o gpurun_out/conv9_pair_full python bench.py --workload conv9 --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_conv9.log 2>&1; echo ncu=$?
