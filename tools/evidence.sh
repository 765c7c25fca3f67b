#!/bin/bash
# Round evidence on the GPU box: default bench line, per-config lines, reference arm, ncu launch
# list of the default bench command, ncu --set full of the blocked kernel (C3 and a C5 sample).
cd "$(dirname "$0")/.."
O=gpurun_out/ev; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 900 python bench.py > $O/bench_C5_default.json 2> $O/bench_C5_default.err
for c in C1 C2 C3 C4; do timeout 300 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.json 2>> $O/bench_err.txt; done
timeout 600 python bench.py --impl reference > $O/bench_C5_reference_arm.json 2>> $O/bench_err.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -c 400 --csv --log-file $O/ncu_launches_C5.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > $O/ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_blocked3 -s 1 -c 1 -o $O/ncu_full_C3 \
  env REPS=2 python tools/cfgtime.py C3 > $O/ncu_full_C3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:potrf_blocked3 -s 1 -c 1 -o $O/ncu_full_C5s \
  python bench.py --config C5 --batch-limit 1500 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > $O/ncu_full_C5s.log 2>&1
