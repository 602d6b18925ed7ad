cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_conv.py tests/test_gpu_p2p.py -x -q --timeout 600 > gpurun_out/pytest_conv_r24.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_conv_r24.log
for v in main pair_dorder; do
  L=""; [ $v != main ] && L=exp/$v/libmapsm.so
  MAPSM_LIB=$L timeout 300 python bench.py --workload conv9 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_conv9_r24_$v.json 2>>gpurun_out/v.err; echo $v $(python -c "import json;d=json.load(open('gpurun_out/bench_conv9_r24_$v.json'));r=d['roofline'];print(d['value'], r.get('kernel_ms_per_launch'), r['frac'], r.get('fma_frac_at_sampled_clock'), d['clocks'])")
done
ncu --set full --import-source on -k regex:conv_tma_kernel -s 6 -c 1 -o gpurun_out/conv9_pairm_full python bench.py --workload conv9 --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_conv9.log 2>&1; echo ncu=$?
