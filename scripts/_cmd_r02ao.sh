# ncu with source: the tail of the pass (scan, placement + write-out), headline
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"k_place_write|k_scan_lb" -c 2 \
  -o gpurun_out/r02ao_tail python scripts/prof_run.py headline > gpurun_out/r02ao_tail.log 2>&1
tail -1 gpurun_out/r02ao_tail.log
