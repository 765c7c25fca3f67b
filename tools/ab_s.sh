#!/bin/bash
# A/B of SPOTRF builds (development): FFMA microbench, then C3/C5 in FP32 with each library
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
./tools/ffma_bench
for lib in paper_conf_ipps_abdelfattahhtd16_b200/libvbatched.so $AB_LIBS; do
  echo "== $lib"
  VBATCHED_LIB=$PWD/$lib QB_ARGS="--precision s" bash tools/quickbench.sh $AB_CFGS
done
