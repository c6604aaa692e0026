timeout 900 python -m pytest -x -q tests/test_gpu_ir.py 2>&1 | tail -2
BEAST_IR_TRACE=1 python scripts/ir_time.py headline b200_D 2>&1 | tail -40
for w in b200_S b200_D b200_C; do python scripts/shard_stats.py $w 8 10; python scripts/shard_stats.py $w 4 10; done
