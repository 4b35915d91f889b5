cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-rX}
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 5 --cpu-seconds 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
for c in transformer_2dev nmt4_2dev_commheavy transformer_4dev_8gpu; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 -o gpurun_out/prof_${TAG}_inception python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_${TAG}.log 2>&1
