set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -6
timeout 600 python bench.py > gpurun_out/r01e_bench_default.json 2> gpurun_out/r01e_bench_default.err; tail -c 3000 gpurun_out/r01e_bench_default.json
timeout 300 python bench.py --workload b200_S --no-cpu-baseline --no-sweep --no-ir > gpurun_out/r01e_bench_b200_S.json 2> gpurun_out/r01e_b200S.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r01e_ref.json 2>&1; tail -c 1500 gpurun_out/r01e_ref.json
