cd $GRAFT_REPO_ROOT
./tools/pipebench3 > gpurun_out/pipebench3.txt 2>&1; cat gpurun_out/pipebench3.txt
timeout 1500 python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/pytest_gpu_r22.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu_r22.log
timeout 600 python bench.py > gpurun_out/bench_default_r22.json 2>gpurun_out/bench_default_r22.err; echo bench=$?; cat gpurun_out/bench_default_r22.json
for w in conv9 conv5; do
timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_${w}_r22.json 2>>gpurun_out/v.err; echo $w $(python -c "import json;d=json.load(open('gpurun_out/bench_${w}_r22.json'));r=d['roofline'];print(d['value'], r.get('kernel_ms_per_launch'), r['frac'], r.get('fma_frac_at_sampled_clock'))")
done
timeout 120 python -c "import __graft_entry__ as g; g.smoke()"; echo smoke=$?
