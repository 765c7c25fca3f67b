#!/bin/bash
# compute-sanitizer on the code changed late in round 2 (vbatched BLAS tile lookup / C prefetch,
# two-level GETRF): memcheck, synccheck, racecheck on the LU, QR and host cases, memcheck on the
# mixed Cholesky batch (KREV). Logs -> gpurun_out/san2/.
cd "$(dirname "$0")/.."
O=gpurun_out/san2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for tool in memcheck synccheck racecheck; do
  for case in lu qr host; do
    timeout 900 compute-sanitizer --tool $tool --report-api-errors no --kernel-name kns=_ZN2vb \
      --error-exitcode 9 python tools/sanitize_case.py $case > $O/${tool}_${case}.log 2>&1
    echo "$tool $case rc=$?" | tee -a $O/summary.txt
  done
done
timeout 900 compute-sanitizer --tool memcheck --report-api-errors no --kernel-name kns=_ZN2vb \
  --error-exitcode 9 python tools/sanitize_case.py mixed > $O/memcheck_mixed.log 2>&1
echo "memcheck mixed rc=$?" | tee -a $O/summary.txt
