cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/e2ex.log
for cfg in ${CFGS:-"2 0" "4 0" "6 0" "8 0"}; do
  set -- $cfg
  if [ $2 = 0 ]; then C=""; else C=$2; fi
  e=$(PESTO_E2E_BUFFERS=$1 PESTO_EVAL32_CPL=$C timeout 300 python bench.py --steps 10 --warmup 4 --no-cpu-baseline 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('e2e', round(d['e2e']['value']/1e6,3), 'search', round(d['value']/1e6,3))" 2>&1)
  echo "buffers=$1 cpl=$2 $e" >> gpurun_out/e2ex.log
done
