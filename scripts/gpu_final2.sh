cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-r1h}
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.log 2>&1; echo "ref rc=$?" >> gpurun_out/bench_ref.log
for c in transformer_2dev nmt4_2dev_commheavy transformer_4dev_8gpu; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1; done
for CFG in inception_v3_2dev transformer_2dev nmt4_2dev_commheavy; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 -o gpurun_out/prof_${TAG}_${CFG} python bench.py --config $CFG --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_${TAG}_${CFG}.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_${CFG}.csv python bench.py --config $CFG --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_${TAG}_${CFG}.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_default.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_${TAG}_default.log 2>&1
