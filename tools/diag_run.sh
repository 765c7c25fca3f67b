#!/bin/bash
# Development diagnostics on the GPU box: timeline build + per-config timelines + uniform sweep.
cd "$(dirname "$0")/.."
python -c "import __graft_entry__ as g; g.build()" >/dev/null
NV=/usr/local/cuda/bin/nvcc
$NV -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
  -cudart shared -DVB_TIMELINE -I include -o build_tl.so paper_conf_ipps_abdelfattahhtd16_b200/csrc/*.cu
timeout 300 python tools/timeline.py build_tl.so ${TL_CFGS:-C2 C3 C4}
timeout 300 python tools/uniform_bench.py ${UB_SIZES:-64x20000 128x10000 192x6000 256x4000 288x3000 320x3000 384x3000 448x2000 512x2000 1024x600}
