# tiled evaluation (k_tile_eval) vs the global flattener: parity, then A/B timings
mkdir -p gpurun_out
timeout 600 python scripts/gpu_quick.py tiny micro headline 2>&1 | tail -12
SWITCHES="BEAST_FLATTENER=1" bash scripts/bench_pair.sh r02af_h --no-sweep --no-ir
SWITCHES="BEAST_FLATTENER=1" bash scripts/bench_pair.sh r02af_S --workload b200_S --steps 10 --no-sweep --no-ir
