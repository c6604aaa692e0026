# tuple words (prefix, m_a, m_b): parity + timing
mkdir -p gpurun_out
timeout 600 python scripts/gpu_quick.py tiny micro headline 2>&1 | grep -E "count|equal|Error" | tail -8
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py tests/test_gpu_fused_gather.py 2>&1 | tail -2
bash scripts/ab2.sh "headline b200_S"
