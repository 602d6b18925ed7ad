cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_task.py tests/test_gpu_histogram.py -x -q --timeout 600 > gpurun_out/pytest_task.log 2>&1; echo pytest=$?; tail -30 gpurun_out/pytest_task.log
for w in life64k conv5; do
  timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --deep-halo 0 --no-cpu-baseline > gpurun_out/bench_$w.json 2>> gpurun_out/bench.err; echo bench_$w=$?; python -c "import json;d=json.load(open('gpurun_out/bench_$w.json'));print(d['value'], d['roofline']['frac'], json.dumps(d.get('chained_task')))"
done
tail -5 gpurun_out/bench.err
