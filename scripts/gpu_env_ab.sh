# A/B of environment settings on the default build: explicit-row device times and the default
# bench line (e2e included) per setting in $ENVS (space-separated, each "A=1,B=2" or "none")
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-envab}
: > gpurun_out/${TAG}.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "${PK:-tiny12 or random_dags or saturated or full_size_sampled or async}" > gpurun_out/${TAG}_pytest.log 2>&1
echo "parity rc=$? $(tail -1 gpurun_out/${TAG}_pytest.log)" >> gpurun_out/${TAG}.log
for rep in 1 2; do
  for v in ${ENVS:-none}; do
    envs=""; [ "$v" != none ] && envs=$(echo $v | tr ',' ' ')
    for c in transformer_2dev inception_v3_2dev; do
      r=$(env $envs timeout 300 python scripts/time_rows.py $c 2>&1 | tail -1 | cut -c1-110)
      echo "$v $r" >> gpurun_out/${TAG}.log
    done
    r=$(env $envs timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],3), 'e2e', round(d['e2e']['value']/1e6,3))" 2>&1)
    echo "$v bench $r" >> gpurun_out/${TAG}.log
  done
done
echo done >> gpurun_out/${TAG}.log
