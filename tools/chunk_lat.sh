#!/bin/bash
# ring-latency records of the blocked kernel (development): bash tools/chunk_lat.sh
cd "$(dirname "$0")/.."
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
  -cudart shared -DVB_CHUNK_LAT -I include -o build_lat.so paper_conf_ipps_abdelfattahhtd16_b200/csrc/*.cu
for c in u1024x600 u512x2000 C5; do timeout 300 python tools/chunk_lat.py build_lat.so $c; done
