# fast-walk check: full GPU parity file + multirank, then the A/B bench (new vs nofast)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-fw}
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -x --durations=15 > gpurun_out/${TAG}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest.log
PK="search_candidate_keys" VARS="nofast" CONFIGS="transformer_2dev inception_v3_2dev nmt4_2dev_commheavy" TAG=${TAG}_ab bash scripts/gpu_abn.sh
