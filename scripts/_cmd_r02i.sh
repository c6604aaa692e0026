for v in "" variants/rc0.so variants/rc512.so variants/rc1024.so; do
  echo "== ${v:-default (256)}"
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_S 8 2>&1 | tail -3
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_C 8 2>&1 | tail -1
  BEAST_LIB_PATH=$v python scripts/shard_time.py headline 20 2>&1 | tail -1
done
