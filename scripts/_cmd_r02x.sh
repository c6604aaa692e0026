timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "headline or full_size or async or host or capacity" tests/test_gpu_fused_gather.py tests/test_gpu_ir.py tests/test_gpu_bench.py 2>&1 | tail -2
bash scripts/ab2.sh "headline b200_S b200_C" variants/nosplit.so
for w in b200_S b200_C; do python bench.py --workload $w --no-cpu-baseline --no-sweep --no-ir --steps 30 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$w', d['write_out']['avg_launch_ms'], d['write_out']['frac'])"; done
python scripts/ir_time.py headline 2>&1 | tail -1
