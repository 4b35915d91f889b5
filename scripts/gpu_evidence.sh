# round-2 evidence pass: ncu capture of K1 (transformer_2dev) + launch list of the default bench,
# sanitizers on the TMA/mbarrier ring, bases after 100 steps (f1 study), host coarsening times
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-r2e}
CFG=${CFG:-transformer_2dev}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 2 -c 1 \
  -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --steps 1 --warmup 2 --no-cpu-baseline --no-e2e \
  > gpurun_out/ncu_full_${TAG}_${CFG}.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_default.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline \
  > gpurun_out/ncu_launch_${TAG}_default.log 2>&1
timeout 600 python tests/tools/dump_bases.py inception_v3_2dev gpurun_out/bases_inception_v3_2dev.npz 0 100 \
  > gpurun_out/dump_bases.log 2>&1
timeout 600 python tests/tools/dump_bases.py transformer_2dev gpurun_out/bases_transformer_2dev.npz 0 100 \
  >> gpurun_out/dump_bases.log 2>&1
timeout 600 python tests/tools/coarsen_time.py gpurun_out/coarsen_time.json > gpurun_out/coarsen_time.log 2>&1
[ -n "$SAN" ] && bash scripts/gpu_sanitize.sh
echo done
