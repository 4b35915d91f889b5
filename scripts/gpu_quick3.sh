cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
for v in base nh; do
  if [ $v = base ]; then L=""; else L=paper_conf_middleware_hafeezsg021_b200/libpesto_$v.so; fi
  for c in inception_v3_2dev transformer_2dev; do
    r=$(PESTO_LIB=$L timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
    echo "$v $c $r" >> gpurun_out/quick.log
  done
done
