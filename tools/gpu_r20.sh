cd $GRAFT_REPO_ROOT
for v in c3_ry2_b3 c3_ry4_n3 c3_ry2_b4; do
  MAPSM_LIB=exp/$v/libmapsm.so timeout 300 python bench.py --workload conv3d --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/v_$v.json 2>>gpurun_out/v.err; echo $v $(python -c "import json;d=json.load(open('gpurun_out/v_$v.json'));print(d['value'], d['roofline']['kernel_ms_per_launch'])")
done
timeout 300 python bench.py --workload conv3d --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/v_base.json 2>>gpurun_out/v.err; echo base $(python -c "import json;d=json.load(open('gpurun_out/v_base.json'));print(d['value'], d['roofline']['kernel_ms_per_launch'])")
for v in c3_r2_ry1_b4 c3_r2_ry2_b3; do
  MAPSM_LIB=exp/$v/libmapsm.so timeout 300 python bench.py --workload conv3d5 --steps 2 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/v_$v.json 2>>gpurun_out/v.err; echo $v $(python -c "import json;d=json.load(open('gpurun_out/v_$v.json'));print(d['value'], d['roofline']['kernel_ms_per_launch'], d['roofline']['fma_frac_at_sampled_clock'])")
done
timeout 300 python bench.py --workload conv3d5 --steps 2 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/v_base5.json 2>>gpurun_out/v.err; echo base5 $(python -c "import json;d=json.load(open('gpurun_out/v_base5.json'));print(d['value'], d['roofline']['kernel_ms_per_launch'], d['roofline']['fma_frac_at_sampled_clock'])")
timeout 600 python bench.py --workload sgemm8k --steps 3 --warmup 2 > gpurun_out/bench_sgemm8k.json 2>>gpurun_out/v.err; cat gpurun_out/bench_sgemm8k.json
tail -3 gpurun_out/v.err
