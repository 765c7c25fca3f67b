#!/bin/bash
# ncu --set full of the small kernel on C2 (one bench step), source-level stall reasons
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:potrf_small -s 2 -c 1 \
  -o gpurun_out/ncu_small_C2 python bench.py --config C2 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --clock-soak 0 > gpurun_out/ncu_small.log 2>&1
echo rc=$?
