#!/bin/bash
# quick GPU iteration: gq.sh "<pytest -k expr or empty>" "<configs>" [extra cmd]
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
if [ -n "$1" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$1" > gpurun_out/pytest_q.txt 2>&1
  echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q.txt
fi
[ -n "$2" ] && bash tools/quickbench.sh $2
[ -n "$3" ] && eval "$3"
true
