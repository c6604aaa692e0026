#!/bin/bash
# usage (on the GPU box): scripts/gpu_iter.sh TAG [workloads...] — gpu tests, bench lines, one k_eval ncu source capture
TAG=${1:-it}; shift
WLS=${@:-headline}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for WL in $WLS; do
  timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --steps 100 > gpurun_out/${TAG}_${WL}.json 2> gpurun_out/${TAG}_${WL}.err
  python - gpurun_out/${TAG}_${WL}.json <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[1]))
    print(d["config"]["workload"], "ms/step %.4f" % d["ms_per_step"], "pts/s %.3e" % d["value"], "frac %.4f" % d["roofline"]["frac"],
          "keval_ms %.4f" % d["roofline"]["avg_launch_ms"], "stages", ["%.4f" % x for x in d.get("stages_ms", [])],
          "fact_ms %.4f" % d["factorised"]["ms_per_step"], "e2e %.3e" % d["e2e"]["value"], d["clocks"])
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
if [ -n "$NCU" ]; then
  WL=${NCU}
  timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_eval -c 1 -o gpurun_out/${TAG}_keval python scripts/prof_run.py $WL > gpurun_out/${TAG}_ncu.log 2>&1
  ncu -i gpurun_out/${TAG}_keval.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_keval_sass.csv 2>&1
  ncu -i gpurun_out/${TAG}_keval.ncu-rep --page raw --csv > gpurun_out/${TAG}_keval_raw.csv 2>&1
fi
echo iter done
