# full round check: smoke, the whole GPU suite (durations), default bench + reference arm, then
# the evidence pass (scripts/gpu_evidence.sh)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-r2f}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 3000 python -m pytest tests -m gpu -q -x --durations=30 > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/${TAG}_bench_ref.log 2>&1; echo "ref rc=$?" >> gpurun_out/${TAG}_bench_ref.log
for c in inception_v3_2dev nmt4_2dev_commheavy transformer_4dev_8gpu; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_$c.log 2>&1
done
TAG=$TAG bash scripts/gpu_evidence.sh
echo done
