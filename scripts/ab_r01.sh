#!/bin/bash
# usage (on the GPU box): scripts/ab_r01.sh — same-box A/B: round-1 tree (variants/r01) vs current, b200_S and headline
for WL in b200_S headline; do
  (cd variants/r01 && timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 100 > ../../gpurun_out/abr01_old_$WL.json 2>/dev/null)
  timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 100 > gpurun_out/abr01_new_$WL.json 2>/dev/null
  for v in old new; do python -c "
import json; d=json.load(open('gpurun_out/abr01_${v}_$WL.json')); print('$v', '$WL', 'ms %.4f'%d['ms_per_step'], 'keval %.4f'%d['roofline']['avg_launch_ms'], ['%.4f'%x for x in d['stages_ms']])"; done
done
