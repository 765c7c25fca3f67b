#!/bin/bash
# Round-2 final evidence on the GPU box -> gpurun_out/ev4/ (summaries copied to profiles/r02/).
cd "$(dirname "$0")/.."
O=gpurun_out/ev4; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_C5_default.json 2> $O/bench_C5_default.err
for c in C1 C2 C3 C4; do timeout 300 python bench.py --config $c --no-cpu-baseline --steps 20 > $O/bench_$c.json 2>> $O/bench_err.txt; done
timeout 300 python bench.py --config C5 --precision s --no-cpu-baseline > $O/bench_C5_spotrf.json 2>> $O/bench_err.txt
timeout 600 python bench.py --impl reference > $O/bench_C5_reference_arm.json 2>> $O/bench_err.txt
VB_BENCH_SHARE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_C5_share_gpu_n2.json 2> $O/bench_share.err
timeout 300 python tools/getrf_bench.py 3000 512 2000 256 > $O/getrf_bench.jsonl 2>> $O/bench_err.txt
OP=qr timeout 300 python tools/getrf_bench.py 3000 512 2000 256 > $O/geqrf_bench.jsonl 2>> $O/bench_err.txt
timeout 300 python tools/zpotrf_bench.py z 3000 512 c 3000 512 z 2000 128 > $O/zpotrf_bench.jsonl 2>> $O/bench_err.txt
timeout 300 python tools/blas_bench.py > $O/blas_bench.jsonl 2>> $O/bench_err.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -c 400 --csv --log-file $O/ncu_launches_C5.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --clock-soak 0 > $O/ncu_bench.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -c 400 --csv --log-file $O/ncu_launches_C2.csv python bench.py --config C2 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --clock-soak 0 > $O/ncu_bench_C2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:potrf_blocked3 -s 1 -c 1 -o $O/ncu_full_C5s \
  python bench.py --config C5 --batch-limit 1500 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --clock-soak 0 > $O/ncu_full_C5s.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:potrf_small -s 2 -c 1 -o $O/ncu_full_C2_small \
  python bench.py --config C2 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --clock-soak 0 > $O/ncu_full_C2.log 2>&1
echo done > $O/DONE
