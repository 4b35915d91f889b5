cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python scripts/time_explicit.py inception_v3_2dev > gpurun_out/texp.log 2>&1
timeout 300 python scripts/time_explicit.py transformer_4dev_8gpu >> gpurun_out/texp.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_explicit.csv python scripts/time_explicit.py inception_v3_2dev > gpurun_out/texp_ncu.log 2>&1
