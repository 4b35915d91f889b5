# A/B of eval32 variants: default lib vs libpesto_$B.so (PESTO_LIB), 2 reps each, --steps 10
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
B=${B:-b0}
: > gpurun_out/ab.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coarse_moves.py -q -x > gpurun_out/pytest_ab.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab.log
for c in ${CONFIGS:-inception_v3_2dev transformer_2dev}; do
 for rep in 1 2; do
  for v in new $B; do
   if [ $v = new ]; then L=""; else L=paper_conf_middleware_hafeezsg021_b200/libpesto_$v.so; fi
   r=$(PESTO_LIB=$L timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],3))" 2>&1)
   echo "$c $v $r" >> gpurun_out/ab.log
  done
 done
done
