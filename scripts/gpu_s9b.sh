cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_coarse_moves.py -q -x > gpurun_out/pytest_s9.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_s9.log
: > gpurun_out/quick.log
for c in ${CONFIGS:-inception_v3_2dev transformer_2dev nmt4_2dev_commheavy transformer_4dev_8gpu}; do
  for cp in 0 20; do
  r=$(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --coarse-pct $cp 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2), d['search']['best_makespans'])" 2>&1)
  echo "$c coarse=$cp $r" >> gpurun_out/quick.log
  done
done
