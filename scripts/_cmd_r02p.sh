python scripts/shard_time.py b200_S 8 2>&1 | tail -3
python scripts/shard_time.py b200_C 8 2>&1 | tail -1
python scripts/shard_time.py b200_D 8 2>&1 | tail -1
python scripts/shard_time.py headline 20 2>&1 | tail -1
python scripts/shard_time.py widened256_b200 10 2>&1 | tail -1
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "virtual or fuzz_shards" tests/test_gpu_fused_gather.py 2>&1 | tail -2
BEAST_IR_TRACE=1 python scripts/ir_time.py headline 2>&1 | tail -16
