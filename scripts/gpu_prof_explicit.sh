cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python scripts/time_explicit.py inception_v3_2dev > gpurun_out/time_explicit.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 -o gpurun_out/prof_explicit python scripts/time_explicit.py inception_v3_2dev > gpurun_out/ncu_explicit.log 2>&1
