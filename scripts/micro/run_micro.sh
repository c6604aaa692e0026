#!/bin/bash
# usage (on the GPU box): scripts/micro/run_micro.sh OUTDIR — integer-pipe and
# packed-scan microbenchmarks (pipes.cu, scan.cu) with the SM clock sampled by
# nvidia-smi during the runs (the printed rates assume the max clock; the log
# carries the observed one).
OUT=$(realpath -m "${1:-gpurun_out}")
mkdir -p "$OUT"
cd "$(dirname "$0")"
[ -x pipes ] || nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o pipes pipes.cu
[ -x scan ] || nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scan scan.cu
nvidia-smi --query-gpu=timestamp,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv -lms 50 > "$OUT/micro_clocks.csv" &
SMI=$!
sleep 0.5
for i in 1 2 3; do echo "== pipes run $i"; ./pipes; done > "$OUT/micro_pipes.txt" 2>&1
for i in 1 2; do echo "== scan run $i"; ./scan; done > "$OUT/micro_scan.txt" 2>&1
kill $SMI
nvidia-smi -q -d CLOCK > "$OUT/micro_clock_q.txt" 2>&1
echo micro done
