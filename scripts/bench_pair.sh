#!/bin/bash
# usage (on the GPU box): scripts/bench_pair.sh TAG [extra bench args] — prints ms/step, frac, stages
# for the default build and for each BEAST_* switch given in $SWITCHES.
TAG=$1; shift
for sw in "" $SWITCHES; do
  env $sw timeout 300 python bench.py --steps 100 --no-cpu-baseline "$@" > gpurun_out/${TAG}_${sw:-default}.json 2> gpurun_out/${TAG}_${sw:-default}.err
  python - "$sw" gpurun_out/${TAG}_${sw:-default}.json <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[2]))
    print(sys.argv[1] or "default", "ms/step %.4f" % d["ms_per_step"], "frac %.4f" % d["roofline"]["frac"],
          "keval %.4f" % d["roofline"]["avg_launch_ms"], "stages", ["%.4f" % x for x in d.get("stages_ms", [])])
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
