cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/cplcheck.log
for rep in 1 2; do
 for cpl in 1 2; do
  r=$(PESTO_EVAL32_CPL=$cpl timeout 300 python bench.py --config inception_v3_2dev --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],3))" 2>&1)
  echo "inception cpl=$cpl $r" >> gpurun_out/cplcheck.log
  r=$(PESTO_EVAL32_CPL=$cpl timeout 300 python scripts/time_explicit.py inception_v3_2dev 2>&1 | head -1)
  echo "explicit cpl=$cpl $r" >> gpurun_out/cplcheck.log
 done
done
