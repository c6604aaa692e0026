timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or full_size or fuzz or virtual or golden" 2>&1 | tail -2
bash scripts/ab2.sh "headline b200_S" variants/pf0.so variants/noF.so
bash scripts/ab2.sh "headline" variants/pf0.so variants/noF.so
