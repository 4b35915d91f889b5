# A/B of the e2e (double-buffered explicit rows) line: default lib vs libpesto_$B.so
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
B=${B:-co}
: > gpurun_out/abe.log
for rep in 1 2; do
 for v in new $B; do
  if [ $v = new ]; then L=""; else L=paper_conf_middleware_hafeezsg021_b200/libpesto_$v.so; fi
  e=$(PESTO_LIB=$L timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('e2e', round(d['e2e']['value']/1e6,3), 'search', round(d['value']/1e6,3))" 2>&1)
  r=$(PESTO_LIB=$L timeout 300 python scripts/time_explicit.py inception_v3_2dev 2>&1 | head -1)
  echo "$v $e | $r" >> gpurun_out/abe.log
 done
done
