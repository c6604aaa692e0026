timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or full_size or fuzz_shards or virtual or wide" tests/test_gpu_fused_gather.py 2>&1 | tail -3
bash scripts/ab2.sh "b200_S headline" variants/l5flat0.so variants/un4ki10.so variants/un4cu2.so variants/un4cu8.so variants/un3.so variants/un8.so
