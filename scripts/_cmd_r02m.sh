for v in "" variants/cc0.so variants/cc512.so variants/cc2048.so; do
  echo "== ${v:-default (cand 128)}"
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_S 8 2>&1 | tail -2
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_C 8 2>&1 | tail -1
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_D 8 2>&1 | tail -1
done
