#!/bin/bash
# Development profiling pass (GPU box): size sweep, phase timers, diagonal-block latency.
# Usage: bash tools/profile_phases.sh > gpurun_out/phases.txt
set -x
cd "$(dirname "$0")/.."
python -c "import __graft_entry__ as g; g.build()" >/dev/null
NV=/usr/local/cuda/bin/nvcc
$NV -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
  -cudart shared -DVB_PHASE_PROF -I include -o build_phase.so paper_conf_ipps_abdelfattahhtd16_b200/csrc/*.cu
$NV -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o tools/diag_bench tools/diag_bench.cu
timeout 120 ./tools/diag_bench
timeout 300 python tools/uniform_bench.py 48x20000 64x20000 96x10000 128x10000 160x6000 192x6000 256x4000 320x3000 384x3000 448x2000 512x2000 640x1000 768x1000 1024x600
for c in C2 C3 C4 u384x3000 u512x2000 u1024x600; do
  SMALL=$([ $c = C2 ] && echo 1) timeout 120 python tools/phase_prof.py build_phase.so $c
done
