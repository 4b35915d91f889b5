cd $GRAFT_REPO_ROOT
PK="search_candidate_keys or multiwave or committed_swaps or search_full_size_parity or wide_eval32" VARS="dt" CONFIGS="transformer_2dev inception_v3_2dev nmt4_2dev_commheavy" TAG=it2_ab bash scripts/gpu_abn.sh
SAN=1 bash scripts/gpu_sanitize.sh
