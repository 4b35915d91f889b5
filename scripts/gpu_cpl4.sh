cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/cpl4.log
PESTO_EVAL32_CPL=4 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "multiwave or search_full_size or wide_eval32" > gpurun_out/pytest_cpl4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_cpl4.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "multiwave" >> gpurun_out/pytest_cpl4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_cpl4.log
for c in transformer_2dev transformer_4dev_8gpu nmt4_2dev_commheavy; do
 for v in base c4 m5 m3; do
  case $v in base) E=""; L="";; c4) E=4; L="";; m5) E=4; L=paper_conf_middleware_hafeezsg021_b200/libpesto_m5.so;; m3) E=4; L=paper_conf_middleware_hafeezsg021_b200/libpesto_m3.so;; esac
  r=$(PESTO_EVAL32_CPL=$E PESTO_LIB=$L timeout 300 python bench.py --config $c --steps 6 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
  echo "$c $v $r" >> gpurun_out/cpl4.log
 done
done
