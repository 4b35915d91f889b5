# end-of-round pass: smoke, the whole GPU suite, every config's bench line, the reference arm,
# host->device bandwidth (the e2e bound), ncu capture of K1 + the default command's launch list,
# sanitizers.  Outputs gpurun_out/${TAG}_*; summarised into profiles/ by hand.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=${TAG:-r2z}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${TAG}_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 3000 python -m pytest tests -m gpu -q -x --durations=15 > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/${TAG}_bench_ref.log 2>&1; echo "ref rc=$?" >> gpurun_out/${TAG}_bench_ref.log
for c in inception_v3_2dev nmt4_2dev_commheavy transformer_4dev_8gpu; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_$c.log 2>&1
done
timeout 300 python - > gpurun_out/${TAG}_h2d.log 2>&1 <<'PY'
import torch
n = 2550136832 // 4
h = torch.empty(n, dtype=torch.int32, pin_memory=True)
d = torch.empty(n, dtype=torch.int32, device="cuda")
for _ in range(2):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    d.copy_(h, non_blocking=True)
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 5
print({"h2d_bytes": n * 4, "ms": ms, "GBps": n * 4 / ms / 1e6})
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 2 -c 1 \
  -o gpurun_out/prof_${TAG}_transformer_2dev python bench.py --config transformer_2dev --steps 1 --warmup 2 --no-cpu-baseline --no-e2e \
  > gpurun_out/ncu_full_${TAG}_transformer_2dev.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_default.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline \
  > gpurun_out/ncu_launch_${TAG}_default.log 2>&1
# the explicit-row (e2e) kernels: device times, K1 mode 0 and K5 captures
for c in transformer_2dev inception_v3_2dev; do
  timeout 300 python scripts/time_rows.py $c >> gpurun_out/${TAG}_rows.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval32_kernel -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_rows python scripts/time_rows.py transformer_2dev > gpurun_out/ncu_${TAG}_rows.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:transpose -s 1 -c 1 \
  -o gpurun_out/prof_${TAG}_k5 python scripts/time_rows.py transformer_2dev > gpurun_out/ncu_${TAG}_k5.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}_rows.csv python scripts/time_rows.py transformer_2dev > /dev/null 2>&1
# the launcher path the driver's scaling run uses (torchrun, env rendezvous), at one rank
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_torchrun.log 2>&1
echo "torchrun rc=$?" >> gpurun_out/${TAG}_torchrun.log
[ -n "$SAN" ] && bash scripts/gpu_sanitize.sh
echo done
