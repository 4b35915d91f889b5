cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for cpl in 2 4 1; do
  PESTO_EVAL32_CPL=$cpl python paper_conf_middleware_hafeezsg021_b200/build.py --force > /dev/null 2>&1
  for c in inception_v3_2dev transformer_2dev transformer_4dev_8gpu; do
    timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/cpl${cpl}_$c.log 2>&1
  done
done
