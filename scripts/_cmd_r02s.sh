timeout 900 python -m pytest -x -q tests/test_gpu_parity.py -k "tiny or micro or headline or full_size or fuzz or virtual or async or host or capacity" tests/test_gpu_fused_gather.py tests/test_gpu_sweep.py 2>&1 | tail -2
bash scripts/ab2.sh "headline b200_S" variants/l4t0.so
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/r02s_launches.csv python scripts/prof_run.py headline > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/r02s_launches.csv
