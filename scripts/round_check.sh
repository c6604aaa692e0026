#!/bin/bash
# Run ON THE GPU BOX (via gpurun): smoke, the GPU test suite, the default bench
# line, the SGEMM-B200 bench line and the reference arm.  usage: scripts/round_check.sh TAG
TAG=${1:-check}
mkdir -p gpurun_out
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -6
timeout 600 python bench.py > gpurun_out/${TAG}_bench_default.json 2> gpurun_out/${TAG}_bench_default.err; tail -c 3000 gpurun_out/${TAG}_bench_default.json
timeout 600 python bench.py --workload b200_S --no-sweep --no-ir > gpurun_out/${TAG}_bench_b200_S.json 2> gpurun_out/${TAG}_b200S.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_ref.json 2>&1; tail -c 1500 gpurun_out/${TAG}_ref.json
