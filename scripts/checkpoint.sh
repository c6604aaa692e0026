#!/bin/bash
# Run ON THE GPU BOX (via gpurun): full GPU suite + smoke, bench lines (default,
# SGEMM-B200), reference arm, launch list and ncu captures for profiles/.
# usage: scripts/checkpoint.sh TAG
TAG=${1:-ck}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench_default.json 2> gpurun_out/${TAG}_bench_default.err; echo "bench rc=$?"
timeout 600 python bench.py --workload b200_S --no-sweep --no-ir --no-cpu-baseline > gpurun_out/${TAG}_bench_b200_S.json 2> gpurun_out/${TAG}_b200S.err
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err
# launch list of one headline pass (cold, serialised) and full captures
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
  --log-file gpurun_out/${TAG}_headline_launches.csv python scripts/prof_run.py headline > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
  --log-file gpurun_out/${TAG}_b200_S_launches.csv python scripts/prof_run.py b200_S > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"k_tile_eval|k_place_write|k_scan_lb" -c 4 \
  -o gpurun_out/${TAG}_headline_keval python scripts/prof_run.py headline > gpurun_out/${TAG}_ncu_keval.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_seg_level -c 3 \
  -o gpurun_out/${TAG}_headline_seglvl python scripts/prof_run.py headline > gpurun_out/${TAG}_ncu_seglvl.log 2>&1
timeout 900 ncu --set full --clock-control none --profile-from-start off -k regex:k_tile_eval -c 2 \
  -o gpurun_out/${TAG}_b200_S_keval python scripts/prof_run.py b200_S > gpurun_out/${TAG}_ncu_keval_S.log 2>&1
for r in headline_keval headline_seglvl b200_S_keval; do
  ncu -i gpurun_out/${TAG}_$r.ncu-rep --page raw --csv > gpurun_out/${TAG}_${r}_raw.csv 2>/dev/null
done
echo checkpoint done
