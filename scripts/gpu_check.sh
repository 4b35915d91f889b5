# quick correctness pass of the search path (default lib) + multirank + A/B of variants
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-chk}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_coarse_moves.py -q -x --durations=10 \
  -k "${PK:-search or swaps or multiwave or wide or move_stats or sharding or nccl or constraints or two_processes or coarse}" \
  > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
PK="search_candidate_keys" TAG=${TAG}_ab bash scripts/gpu_abn.sh
