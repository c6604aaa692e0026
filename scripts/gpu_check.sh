#!/bin/bash
# usage (on the GPU box): scripts/gpu_check.sh TAG — full -m gpu suite, smoke, default bench line
TAG=${1:-chk}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/${TAG}_pytest.log 2>&1
echo "pytest rc=$?"; tail -5 gpurun_out/${TAG}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
python - gpurun_out/${TAG}_bench.json <<'PY'
import json, sys
d = json.load(open(sys.argv[1]))
print("ms/step %.4f value %.3e frac %.3f frac_scan %.3f keval_ms %.4f count_ms %.4f e2e %.3e" % (
    d["ms_per_step"], d["value"], d["roofline"]["frac"], d["roofline"]["frac_measured_scan"],
    d["roofline"]["avg_launch_ms"], d["count"]["ms_per_step"], d["e2e"]["value"]), d["clocks"])
PY
