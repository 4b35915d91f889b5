# explicit-row path (the e2e leg): parity subset, then device time of K5 + K1 mode 0 per variant
# ($VARS: libpesto_<v>.so builds), launch lists, one ncu capture of K1 mode 0
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-rows2}
L() { [ "$1" = new ] && echo "" || echo paper_conf_middleware_hafeezsg021_b200/libpesto_$1.so; }
for v in new ${PVARS}; do
  PESTO_LIB=$(L $v) timeout 900 python -m pytest tests/test_gpu_parity.py -q -x \
    -k "tiny12 or random_dags or saturated or full_size_sampled or async" > gpurun_out/${TAG}_pytest_$v.log 2>&1
  echo "$v rc=$? $(tail -1 gpurun_out/${TAG}_pytest_$v.log)" >> gpurun_out/${TAG}_ab.log
done
for rep in 1 2; do
  for c in ${CONFIGS:-transformer_2dev inception_v3_2dev}; do
    for v in new $VARS; do
      r=$(PESTO_LIB=$(L $v) timeout 300 python scripts/time_rows.py $c 2>&1 | tail -1)
      echo "$v $r" >> gpurun_out/${TAG}_ab.log
    done
  done
done
for v in new $VARS; do
  PESTO_LIB=$(L $v) timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}_$v.csv python scripts/time_rows.py transformer_2dev > /dev/null 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_rows python scripts/time_rows.py transformer_2dev > gpurun_out/ncu_${TAG}_rows.log 2>&1
[ -n "$NCU2" ] && PESTO_LIB=$(L $NCU2) timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_rows_$NCU2 python scripts/time_rows.py transformer_2dev > gpurun_out/ncu_${TAG}_rows2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:transpose -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_k5 python scripts/time_rows.py transformer_2dev > gpurun_out/ncu_${TAG}_k5.log 2>&1
echo done >> gpurun_out/${TAG}_ab.log
