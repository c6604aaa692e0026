#!/bin/bash
# usage (on the GPU box): scripts/ab2.sh "WL1 WL2" variant.so... — k_eval / step A/B of in-tree variant builds
WLS=$1; shift
for WL in $WLS; do
for v in "" "$@"; do
  BEAST_LIB_PATH=$v timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 60 > gpurun_out/ab.json 2> gpurun_out/ab.err
  python - "${v:-default}" <<'PY'
import json, sys
try:
    d = json.load(open("gpurun_out/ab.json"))
    print("%-22s" % sys.argv[1], "%-9s" % d["config"]["workload"], "ms/step %.4f" % d["ms_per_step"], "frac %.4f" % d["roofline"]["frac"],
          "keval_ms %.4f" % d["roofline"]["avg_launch_ms"], "stages", ["%.4f" % x for x in d.get("stages_ms", [])])
except Exception as e:
    print(sys.argv[1], "FAILED", e, open("gpurun_out/ab.err").read()[-500:])
PY
done
done
