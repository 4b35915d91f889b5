cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --dispatch nondelay --steps 3 --warmup 3 --no-e2e --cpu-seconds 8 > gpurun_out/bench_nd.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_nd_inception.csv python bench.py --dispatch nondelay --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_nd.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nondelay_kernel -s 1 -c 1 -o gpurun_out/prof_nd_inception python bench.py --dispatch nondelay --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_nd.log 2>&1
