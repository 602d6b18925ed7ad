cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_unmodified.py -x -q --timeout 600 > gpurun_out/pytest_unmod.log 2>&1; echo pytest=$?; tail -30 gpurun_out/pytest_unmod.log
for v in c3_ry2_b3 c3_ry4_n3 c3_ry2_b4; do
  if [ -f exp/$v/libmapsm.so ]; then MAPSM_LIB=exp/$v/libmapsm.so timeout 300 python bench.py --workload conv3d --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/v_$v.json 2>>gpurun_out/v.err; echo $v $(python -c "import json;d=json.load(open('gpurun_out/v_$v.json'));print(d['value'], d['roofline']['kernel_ms_per_launch'])"); fi
done
timeout 300 python bench.py --workload conv3d5 --steps 2 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_conv3d5.json 2>>gpurun_out/v.err; python -c "import json;d=json.load(open('gpurun_out/bench_conv3d5.json'));print('conv3d5', d['value'], d['roofline'])"
tail -3 gpurun_out/v.err
