#!/bin/bash
# summarise gpurun_out results (local helper)
tail -3 gpurun_out/pytest_gpu.log
for f in gpurun_out/bench*.log; do python -c "
import json,sys
for l in open('$f'):
    if l.startswith('{'):
        d=json.loads(l); print(d['config']['workload'], round(d['value']), 'cand/s', round(d['ms_per_step'],2),'ms', 'eval', round(d['eval_kernel_ms'],2), 'frac', round(d['roofline']['frac'],3), 'e2e', d['e2e'] and round(d['e2e']['value']))
"; done
