timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or full_size or fuzz or virtual" tests/test_gpu_fused_gather.py tests/test_gpu_sweep.py 2>&1 | tail -3
bash scripts/ab2.sh "b200_S headline" variants/l5flat0.so
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/r02d_launches.csv python scripts/prof_run.py headline > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/r02d_launches.csv
