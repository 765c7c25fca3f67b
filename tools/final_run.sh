#!/bin/bash
# Final validation on the GPU box: smoke, the whole GPU test suite, then tools/evidence.sh.
cd "$(dirname "$0")/.."
python __graft_entry__.py smoke > gpurun_out/final_smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -3 > gpurun_out/final_pytest.txt
bash tools/evidence.sh > gpurun_out/ev.log 2>&1
