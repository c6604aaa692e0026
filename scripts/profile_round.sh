#!/bin/bash
# Run ON THE GPU BOX (via gpurun): launch list of a short bench run and one
# full ncu capture of the dominant kernel k_eval<A>, for profiles/.
# usage: scripts/profile_round.sh TAG [workload]
TAG=${1:-r01}; WL=${2:-headline}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/${TAG}_${WL}_launches.csv \
    python bench.py --steps 3 --warmup 3 --workload $WL --no-cpu-baseline --no-sweep --no-ir > gpurun_out/${TAG}_${WL}_bench_under_ncu.log 2>&1
ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k k_eval -c 1 -o gpurun_out/${TAG}_${WL}_keval \
    python scripts/prof_run.py $WL > gpurun_out/${TAG}_${WL}_ncu_full.log 2>&1
ncu -i gpurun_out/${TAG}_${WL}_keval.ncu-rep --page raw --csv > gpurun_out/${TAG}_${WL}_keval_raw.csv 2>/dev/null
ncu -i gpurun_out/${TAG}_${WL}_keval.ncu-rep --page details > gpurun_out/${TAG}_${WL}_keval_details.txt 2>/dev/null
echo profile done
