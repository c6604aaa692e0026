mkdir -p gpurun_out
timeout 300 python scripts/gpu_quick.py headline 2>&1 | tail -3
BEAST_LIB_PATH=variants/l5first.so timeout 300 python scripts/gpu_quick.py headline 2>&1 | tail -3
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_l5_eval -c 1 \
  -o gpurun_out/r02aj_l5e python scripts/prof_run.py headline > gpurun_out/r02aj_l5e.log 2>&1
tail -2 gpurun_out/r02aj_l5e.log
