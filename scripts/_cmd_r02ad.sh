timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or full_size or fuzz or virtual or async or host or golden" tests/test_gpu_fused_gather.py tests/test_gpu_sweep.py 2>&1 | tail -3
bash scripts/ab2.sh "headline b200_S" variants/noF.so
bash scripts/ab2.sh "headline" variants/noF.so
