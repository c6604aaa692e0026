# ncu with source: the three prefix levels and both tile kernels, headline
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"k_seg_level|k_tile_eval" -c 5 \
  -o gpurun_out/r02am_hl python scripts/prof_run.py headline > gpurun_out/r02am_hl.log 2>&1
tail -1 gpurun_out/r02am_hl.log
