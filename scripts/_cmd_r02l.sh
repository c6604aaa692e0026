for v in "" variants/rc512.so variants/rc1024.so; do
  echo "== ${v:-default (256)}"
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_S 8 2>&1 | tail -3
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_C 8 2>&1 | tail -1
  BEAST_LIB_PATH=$v python scripts/shard_time.py headline 20 2>&1 | tail -1
done
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "virtual or fuzz_shards" tests/test_gpu_fused_gather.py 2>&1 | tail -2
BEAST_IR_TRACE=1 python scripts/ir_time.py headline 2>&1 | tail -40
