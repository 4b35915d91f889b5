# explicit-row fast segment: the explicit-row parity tests, then e2e A/B (new vs norows)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-rows}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nondelay.py -q -x --durations=5 \
  -k "tiny12 or random_dags or saturated or ineligible or full_size_sampled or async or constraints_explicit or congestion_free_links or exhaustive" \
  > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
: > gpurun_out/${TAG}_ab.log
for rep in 1 2; do
  for c in transformer_2dev inception_v3_2dev; do
    for v in new norows; do
      L=""; [ $v != new ] && L=paper_conf_middleware_hafeezsg021_b200/libpesto_$v.so
      r=$(PESTO_LIB=$L timeout 600 python bench.py --config $c --steps 6 --warmup 3 --no-cpu-baseline 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],3), 'e2e', round(d['e2e']['value']/1e6,3))" 2>&1)
      echo "$c $v $r" >> gpurun_out/${TAG}_ab.log
    done
  done
done
echo done >> gpurun_out/${TAG}_ab.log
