cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
for c in inception_v3_2dev transformer_2dev nmt4_2dev_commheavy; do
    r=$(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
    echo "$c $r" >> gpurun_out/quick.log
done
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
