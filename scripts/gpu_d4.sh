# D <= 4 fast walk: parity of every D = 4 / D = 3 search test, then A/B vs the C++ walk
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-d4}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coarse_moves.py tests/test_gpu_multirank.py -q -x --durations=5 \
  -k "search or swaps or multiwave or wide or move_stats or sharding or constraints or coarse or checkpoint or random_dags or full_size" \
  > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
PK="search_candidate_keys" VARS="nod4" CONFIGS="transformer_4dev_8gpu transformer_2dev" TAG=${TAG}_ab bash scripts/gpu_abn.sh
