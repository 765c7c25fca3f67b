#!/bin/bash
# quick per-config bench summary (development tool): quickbench.sh [configs...]
# full JSON lines -> gpurun_out/qb_<cfg>.json
cfgs=${@:-C1 C2 C3 C4 C5}
mkdir -p gpurun_out
for c in $cfgs; do
  timeout 300 python bench.py --config $c --no-e2e --no-cpu-baseline ${QB_ARGS} 2>>gpurun_out/qb_err.log > gpurun_out/qb_$c.json
  python -c "import json,sys; d=json.loads(open('gpurun_out/qb_$c.json').read()); print(d['config']['workload'][:3], round(d['value'],1), d['unit'], round(d['ms_per_step'],4), 'ms', round(d['roofline']['frac'],4), 'kern_ms', round(d['roofline']['kernel_ms'],4), 'clk', d['clocks'].get('sm_mhz'), d['clocks'].get('samples'), d['clocks'].get('reasons'))"
done
