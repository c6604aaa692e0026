# ncu full captures with source: k_tile_eval<A> (tiled) and k_eval<A> (global flattener), headline
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_tile_eval -c 2 \
  -o gpurun_out/r02ag_tile python scripts/prof_run.py headline > gpurun_out/r02ag_tile.log 2>&1
BEAST_FLATTENER=1 timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_eval -c 1 \
  -o gpurun_out/r02ag_keval python scripts/prof_run.py headline > gpurun_out/r02ag_keval.log 2>&1
ls -la gpurun_out/
