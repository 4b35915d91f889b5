cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 2 -c 1 -o gpurun_out/prof_mode0 python scripts/time_explicit.py inception_v3_2dev > gpurun_out/ncu_mode0.log 2>&1
