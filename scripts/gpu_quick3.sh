cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
for c in inception_v3_2dev transformer_2dev; do
  for rep in 1 2; do
    r=$(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,3), round(d['eval_kernel_ms'],2))" 2>&1)
    echo "$c $r" >> gpurun_out/quick.log
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum,launch__grid_size,launch__block_size,launch__registers_per_thread,launch__occupancy_limit_registers,launch__occupancy_limit_shared_mem,sm__warps_active.avg.per_cycle_active --clock-control none -k regex:eval32 -c 2 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_occ.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
