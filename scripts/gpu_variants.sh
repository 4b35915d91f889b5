cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/variants.log
for v in base p4 p5; do
  if [ $v = base ]; then L=""; else L=paper_conf_middleware_hafeezsg021_b200/libpesto_$v.so; fi
  for c in inception_v3_2dev transformer_2dev transformer_4dev_8gpu nmt4_2dev_commheavy; do
      r=$(PESTO_LIB=$L timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
      echo "$v $c $r" >> gpurun_out/variants.log
  done
done
PESTO_LIB=paper_conf_middleware_hafeezsg021_b200/libpesto_p4.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "search or swap or congestion or constraints" > gpurun_out/p4_tests.log 2>&1; echo "rc=$?" >> gpurun_out/p4_tests.log
