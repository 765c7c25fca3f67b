#!/bin/bash
# quick per-config bench summary (development tool): quickbench.sh [configs...]
cfgs=${@:-C1 C2 C3 C4 C5}
for c in $cfgs; do
  timeout 300 python bench.py --config $c --no-e2e --no-cpu-baseline 2>>gpurun_out/qb_err.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'][:3], round(d['value'],1), d['unit'], round(d['ms_per_step'],4), 'ms', round(d['roofline']['frac'],4), 'kern_ms', round(d['roofline']['kernel_ms'],4))"
done
