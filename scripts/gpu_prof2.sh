cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-r1c}
for CFG in inception_v3_2dev transformer_2dev nmt4_2dev_commheavy; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_${TAG}_${CFG}.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_${CFG}.csv python bench.py --config $CFG --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_${TAG}_${CFG}.log 2>&1
done
