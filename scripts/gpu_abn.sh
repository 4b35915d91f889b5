# A/B of eval32 variants (PESTO_LIB): the default lib ("new") vs each entry of $VARS, written
# LIB or LIB@ENV=V,ENV2=V2 (libpesto_LIB.so, "new" = the default lib, plus environment).
# Per variant: the search parity subset, then bench.py --steps 10 on each config, 2 reps.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-ab}
: > gpurun_out/${TAG}.log
run_v() {   # $1 = variant spec, rest = command
  local spec=$1; shift
  local lib=${spec%%@*} envs=""
  [ "$spec" != "$lib" ] && envs=$(echo ${spec#*@} | tr ',' ' ')
  local L=""
  [ "$lib" != new ] && L=paper_conf_middleware_hafeezsg021_b200/libpesto_$lib.so
  env PESTO_LIB=$L $envs "$@"
}
for v in new $VARS; do
  run_v $v timeout 900 python -m pytest tests/test_gpu_parity.py -q -x \
    -k "${PK:-search_candidate_keys or search_steps_match or multiwave or committed_swaps or wide_eval32}" \
    > gpurun_out/${TAG}_pytest_${v//[@=,]/_}.log 2>&1
  echo "$v parity rc=$? $(tail -1 gpurun_out/${TAG}_pytest_${v//[@=,]/_}.log)" >> gpurun_out/${TAG}.log
done
for rep in 1 2; do
 for c in ${CONFIGS:-transformer_2dev nmt4_2dev_commheavy inception_v3_2dev}; do
  for v in new $VARS; do
   r=$(run_v $v timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],3))" 2>&1)
   echo "$c $v $r" >> gpurun_out/${TAG}.log
  done
 done
done
echo done >> gpurun_out/${TAG}.log
