cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coarse_moves.py -q -x > gpurun_out/pytest_nmt4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_nmt4.log
: > gpurun_out/nmt4.log
for rep in 1 2; do
 for c in nmt4_2dev_commheavy inception_v3_2dev; do
  r=$(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],3), d['search']['best_makespans'])" 2>&1)
  echo "$c $r" >> gpurun_out/nmt4.log
 done
done
