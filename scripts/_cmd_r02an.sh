# fused A+B tile kernel (k_tile_eval_ab): parity; A/B vs separate tile kernels
mkdir -p gpurun_out
timeout 600 python scripts/gpu_quick.py tiny micro headline 2>&1 | grep -E "count|equal|Error" | tail -8
for WL in headline b200_S; do for SW in BEAST_FUSE_AB=1 BEAST_FUSE_AB=0; do env $SW timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 60 > gpurun_out/abf.json 2>gpurun_out/abf.err; python -c "
import json; d=json.load(open('gpurun_out/abf.json')); print('$SW'.ljust(20), d['config']['workload'], 'ms/step %.4f'%d['ms_per_step'], 'keval %.4f'%d['roofline']['avg_launch_ms'], ['%.4f'%x for x in d['stages_ms']])" 2>/dev/null || tail -3 gpurun_out/abf.err; done; done
