# k_prefix45 (L4 + L5-L7 in one persistent kernel): parity; A/B vs separate levels; IR trace
mkdir -p gpurun_out
timeout 120 python scripts/gpu_quick.py tiny micro headline 2>&1 | grep -E "count|equal|Error" | tail -8
timeout 400 python -m pytest -x -q tests/test_gpu_parity.py 2>&1 | tail -2
for WL in headline b200_S; do for SW in BEAST_FUSE_PREFIX=1 BEAST_FUSE_PREFIX=0; do env $SW timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 60 > gpurun_out/abf.json 2>gpurun_out/abf.err; python -c "
import json; d=json.load(open('gpurun_out/abf.json')); print('$SW'.ljust(20), d['config']['workload'], 'ms/step %.4f'%d['ms_per_step'], 'keval %.4f'%d['roofline']['avg_launch_ms'], ['%.4f'%x for x in d['stages_ms']])" 2>/dev/null || tail -3 gpurun_out/abf.err; done; done
BEAST_IR_TRACE=1 timeout 600 python scripts/ir_time.py headline 2>&1 | tail -20
