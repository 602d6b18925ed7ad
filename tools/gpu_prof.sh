cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:life_tb_kernel -s 2 -c 1 -o gpurun_out/r01_life64k_tb8 python tools/kbench.py life64k 16 --deep 8 > gpurun_out/ncu1.log 2>&1; echo ncu1=$?
ncu --set full --clock-control none --import-source on -k regex:conv_tma_kernel -s 2 -c 1 -o gpurun_out/r01_conv9 python tools/kbench.py conv9 4 > gpurun_out/ncu2.log 2>&1; echo ncu2=$?
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01_life64k_deep_launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu3.log 2>&1; echo ncu3=$?
