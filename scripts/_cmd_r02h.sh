python scripts/shard_stats.py b200_S 8 10
python scripts/shard_stats.py headline 8 20
python scripts/shard_time.py b200_S 10
