cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool memcheck --show-backtrace device --print-limit 5 python -m pytest tests/test_gpu_parity.py -q -x -k "seed8_n800" > gpurun_out/sanitize.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "seed9 or seed10 or seed11 or seed12 or saturat or ineligible or full_size or search" > gpurun_out/pytest_rest.log 2>&1
