for v in variants/p16.so variants/p8.so; do BEAST_LIB_PATH=$v timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or fuzz_1" 2>&1 | tail -1; done
bash scripts/ab2.sh "headline" variants/p16.so variants/p8.so variants/p16s2.so variants/p32s2.so
