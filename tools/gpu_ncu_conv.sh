cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_tma -s 3 -c 1 -o gpurun_out/prof_conv9 python tools/kbench.py conv9 4 > gpurun_out/ncu_conv9.log 2>&1; echo ncu9=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_tma -s 3 -c 1 -o gpurun_out/prof_conv5 python tools/kbench.py conv5 4 > gpurun_out/ncu_conv5.log 2>&1; echo ncu5=$?
