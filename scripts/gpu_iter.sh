# one iteration: new tests (-k $PK), A/B of $VARS, ncu capture of K1 on $CFG, optional sanitizers
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-it}
CFG=${CFG:-transformer_2dev}
timeout 900 python -m pytest tests -m gpu -q -x -k "${PK:-checkpoint}" > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
[ -n "$VARS" ] && PK="search_candidate_keys" TAG=${TAG}_ab bash scripts/gpu_abn.sh
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 2 -c 1 \
  -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --steps 1 --warmup 2 --no-cpu-baseline --no-e2e \
  > gpurun_out/ncu_full_${TAG}_${CFG}.log 2>&1
[ -n "$SAN" ] && bash scripts/gpu_sanitize.sh
echo done
