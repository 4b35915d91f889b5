cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
for v in base w7; do
  if [ $v = base ]; then L=""; else L=paper_conf_middleware_hafeezsg021_b200/libpesto_$v.so; fi
  for c in inception_v3_2dev; do
   for rep in 1 2; do
    r=$(PESTO_LIB=$L timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2), round(d['e2e']['value']/1e6,3))" 2>&1)
    echo "$v $c $r" >> gpurun_out/quick.log
   done
  done
done
PESTO_LIB=paper_conf_middleware_hafeezsg021_b200/libpesto_w7.so timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_w7.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_w7.log
