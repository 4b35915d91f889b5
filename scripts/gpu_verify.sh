# verification pass of the default build: the GPU suite, the default bench line and the
# inception / transformer_4dev lines, the explicit-row device times
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-ver}
timeout 3000 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
for c in ${CONFIGS:-inception_v3_2dev}; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_$c.log 2>&1
done
for c in transformer_2dev inception_v3_2dev; do
  timeout 300 python scripts/time_rows.py $c >> gpurun_out/${TAG}_rows.log 2>&1
done
echo done
