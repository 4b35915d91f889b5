cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for cpl in ${CPLS:-0 1 2}; do
  for c in ${CONFIGS:-inception_v3_2dev nmt4_2dev_commheavy transformer_2dev}; do
    PESTO_EVAL32_CPL=$cpl timeout 300 python bench.py --config $c --steps 8 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cpl${cpl}_$c.log 2>&1
  done
done
