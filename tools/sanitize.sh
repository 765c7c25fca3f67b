#!/bin/bash
# compute-sanitizer memcheck / synccheck / initcheck / racecheck on the C1 and mixed cases
# (tools/sanitize_case.py). Logs -> gpurun_out/san/ (copied to profiles/r02/ when judged).
cd "$(dirname "$0")/.."
O=gpurun_out/san; mkdir -p $O
for tool in memcheck synccheck initcheck racecheck; do
  for case in c1 mixed lu z; do
    # initcheck must see the writes of the (non-vb::) input generator kernels too, so it runs
    # unfiltered, on a 50-matrix version of the mixed case (the full one exceeds the time limit)
    filt="--kernel-name kns=_ZN2vb"
    arg=$case
    if [ $tool = initcheck ]; then filt=""; [ $case = mixed ] && arg=mixed_small; fi
    # API-call error reports are off: torch's lazy module loading probes cuKernelGetFunction
    # with handles of kernels it has not loaded (CUDA_ERROR_INVALID_HANDLE), unrelated to ours
    extra="--report-api-errors no"
    timeout 900 compute-sanitizer --tool $tool $extra $filt --error-exitcode 9 \
      python tools/sanitize_case.py $arg > $O/${tool}_${case}.log 2>&1
    echo "$tool $case rc=$?" | tee -a $O/summary.txt
  done
done
