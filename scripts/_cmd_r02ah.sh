# tiled evaluation, 512-job tiles + PTX chunk grab: parity; A/B vs 256-job tiles, guide 4, and the global flattener
mkdir -p gpurun_out
timeout 600 python scripts/gpu_quick.py tiny micro headline 2>&1 | grep -v "^ *$" | tail -8
bash scripts/ab2.sh "headline b200_S" variants/tj256.so variants/guide4.so
for WL in headline b200_S; do BEAST_FLATTENER=1 timeout 300 python bench.py --workload $WL --no-cpu-baseline --no-sweep --no-ir --steps 60 > gpurun_out/abf.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/abf.json')); print('FLATTENER', d['config']['workload'], 'ms/step %.4f'%d['ms_per_step'], 'keval %.4f'%d['roofline']['avg_launch_ms'], ['%.4f'%x for x in d['stages_ms']])"; done
