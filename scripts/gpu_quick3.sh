cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "saturation or search or swap" > gpurun_out/pytest_wide.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_wide.log
for c in nmt4_2dev_commheavy inception_v3_2dev transformer_2dev; do
    r=$(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
    echo "$c $r" >> gpurun_out/quick.log
done
