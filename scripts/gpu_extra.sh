cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 1200 python scripts/fig_trends.py --config nmt4_2dev_commheavy --steps 100 > gpurun_out/fig_trends.log 2>&1; echo "rc=$?" >> gpurun_out/fig_trends.log
