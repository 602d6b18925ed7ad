cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_conv.py tests/test_gpu_p2p.py tests/test_gpu_task.py -x -q --timeout 600 > gpurun_out/pytest_r26.log 2>&1; echo pytest=$?; tail -n 2 gpurun_out/pytest_r26.log
MAPSM_LIB=exp/pair_r2/libmapsm.so timeout 600 python -m pytest tests/test_gpu_conv.py -x -q --timeout 600 -k "random_vs_oracle or config4" > gpurun_out/pytest_r26_pair_r2.log 2>&1; echo pytest_pair_r2=$?; tail -n 2 gpurun_out/pytest_r26_pair_r2.log
for v in main pair_r2 main pair_r2; do
  L=""; [ $v != main ] && L=exp/$v/libmapsm.so
  MAPSM_LIB=$L timeout 300 python bench.py --workload conv5 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_conv5_r26_$v.json 2>>gpurun_out/v.err; echo $v $(python -c "import json;d=json.load(open('gpurun_out/bench_conv5_r26_$v.json'));r=d['roofline'];print(d['value'], r.get('kernel_ms_per_launch'), r['frac'], r.get('fma_frac_at_sampled_clock'), d['clocks'])")
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/hist_launches.csv python bench.py --workload hist8k --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/hist_ncu.log 2>&1; echo ncu_hist=$?
timeout 120 python -c "import __graft_entry__ as g; g.smoke()"; echo smoke=$?
