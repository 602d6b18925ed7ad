cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
bash tools/gpu_tune.sh life64k old p2 p3 p4 p6 p3mb3 > gpurun_out/tune_life64k.txt 2>&1
cat gpurun_out/tune_life64k.txt
timeout 900 python -m pytest tests/test_gpu_life.py -x -q > gpurun_out/pytest_life.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_life.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:life_step -s 3 -c 1 -o gpurun_out/prof_life_p3 python tools/kbench.py life64k 4 > gpurun_out/ncu_life.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_life.log
