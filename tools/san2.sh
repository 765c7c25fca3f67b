cd "$(dirname "$0")/.."
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
mkdir -p gpurun_out/san2
for t in "racecheck mixed_gather" "synccheck mixed_gather"; do set -- $t
  timeout 1200 compute-sanitizer --tool $1 --report-api-errors no --kernel-name kns=_ZN2vb --error-exitcode 9 python tools/sanitize_case.py $2 > gpurun_out/san2/$1_$2.log 2>&1; echo "$1 $2 rc=$?"
done
