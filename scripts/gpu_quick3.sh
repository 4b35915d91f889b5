cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
for w in 1 2; do
    r=$(PESTO_WIDE_CPL=$w timeout 300 python bench.py --config nmt4_2dev_commheavy --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | grep '^{' | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
    echo "wide_cpl=$w $r" >> gpurun_out/quick.log
done
