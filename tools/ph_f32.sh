#!/bin/bash
# phase timers of the blocked kernel, FP64 vs FP32 storage (development)
cd "$(dirname "$0")/.."
NV=/usr/local/cuda/bin/nvcc
$NV -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
  -cudart shared -DVB_PHASE_PROF -I include -o build_phase.so paper_conf_ipps_abdelfattahhtd16_b200/csrc/*.cu
for c in ${PH_CFGS:-u512x2000 u1024x600}; do
 for d in f64 f32; do DTYPE=$d timeout 120 python tools/phase_prof.py build_phase.so $c; done
done
