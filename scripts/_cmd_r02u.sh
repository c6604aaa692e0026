timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or fuzz" 2>&1 | tail -2
for v in variants/p64.so variants/p128.so variants/p256.so; do BEAST_LIB_PATH=$v timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or fuzz_1" 2>&1 | tail -1; done
bash scripts/ab2.sh "headline b200_S" variants/p64.so variants/p128.so variants/p256.so
