#!/bin/bash
# usage (on the GPU box): scripts/gpu_iter2.sh TAG [FULL] — parity subset (or the full -m gpu suite
# with FULL=1), headline + SGEMM-B200 bench lines, ncu launch list of one headline pass
TAG=${1:-it}; FULL=${2:-0}
mkdir -p gpurun_out
if [ "$FULL" = "1" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.log 2>&1
else
  timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or full_size or fuzz_shards or virtual or empty or degenerate or async or capacity or host" tests/test_gpu_fused_gather.py tests/test_gpu_sweep.py > gpurun_out/${TAG}_pytest.log 2>&1
fi
echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest.log
for WL in headline b200_S; do
  timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 100 > gpurun_out/${TAG}_${WL}.json 2> gpurun_out/${TAG}_${WL}.err
  python - gpurun_out/${TAG}_${WL}.json <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[1]))
    print(d["config"]["workload"], "ms/step %.4f" % d["ms_per_step"], "pts/s %.3e" % d["value"], "frac %.4f" % d["roofline"]["frac"],
          "keval_ms %.4f" % d["roofline"]["avg_launch_ms"], "count_ms %.4f" % d["count"]["ms_per_step"],
          "write %.4f" % (d["write_out"] or {}).get("avg_launch_ms", -1),
          "stages", ["%.4f" % x for x in d.get("stages_ms", [])], "fact_ms %.4f" % d["factorised"]["ms_per_step"], d["clocks"]["sm_mhz"])
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
  --log-file gpurun_out/${TAG}_launches.csv python scripts/prof_run.py headline > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/${TAG}_launches.csv 2>&1 | tail -25
echo iter done
