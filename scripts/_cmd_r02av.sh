# pipelined prefix levels: parity (quick + parity suite), trace, timing
mkdir -p gpurun_out
timeout 120 python scripts/gpu_quick.py tiny micro headline 2>&1 | grep -E "equal|Error"
timeout 600 python -m pytest -x -q tests/test_gpu_parity.py 2>&1 | tail -2
BEAST_LIB_PATH=variants/trace.so timeout 200 python scripts/tile_trace.py headline 2>&1 | grep -E "^L"
bash scripts/ab2.sh "headline b200_S"
