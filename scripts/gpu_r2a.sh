# round 2, first GPU pass: tests, smoke, default bench (transformer_2dev), reference arm,
# one ncu --set full capture of K1 on transformer_2dev + the default command's launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-r2a}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/${TAG}_bench_ref.log 2>&1; echo "ref rc=$?" >> gpurun_out/${TAG}_bench_ref.log
CFG=transformer_2dev
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 2 -c 1 -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --steps 1 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_${TAG}_${CFG}.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_default.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_${TAG}_default.log 2>&1
echo done
