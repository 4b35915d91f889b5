cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
timeout 900 python -m pytest tests/test_gpu_nondelay.py -q -x > gpurun_out/nd_tests.log 2>&1; echo "rc=$?" >> gpurun_out/nd_tests.log
timeout 300 python scripts/time_nondelay.py inception_v3_2dev 8192 >> gpurun_out/quick.log 2>&1
timeout 300 python bench.py --dispatch nondelay --steps 3 --warmup 2 --no-e2e --no-cpu-baseline 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('nd bench', round(d['value']), d['eval_kernel_ms'])" >> gpurun_out/quick.log
