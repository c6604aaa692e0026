for v in "" variants/rc1024.so variants/rc0.so; do
  echo "== ${v:-default (256)}"
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_S 8 2>&1 | tail -3
  BEAST_LIB_PATH=$v python scripts/shard_time.py b200_C 8 2>&1 | tail -1
  BEAST_LIB_PATH=$v python scripts/shard_time.py headline 20 2>&1 | tail -1
done
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "virtual or fuzz_shards" tests/test_gpu_sweep.py 2>&1 | tail -2
timeout 300 python bench.py --no-cpu-baseline --no-ir --steps 50 > gpurun_out/r02k_bench.json 2>gpurun_out/r02k_bench.err
python -c "import json; d=json.load(open('gpurun_out/r02k_bench.json')); print('sweep', d['sweep']['ms'], d['sweep']['sequential_ms'], d['sweep']['speedup_vs_sequential'], 'step', d['ms_per_step'])"
