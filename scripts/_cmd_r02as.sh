# IR engine: thread-per-parent threshold sweep (headline), parity of the default build
mkdir -p gpurun_out
timeout 120 python scripts/gpu_quick.py tiny micro headline 2>&1 | grep -E "equal|Error" | tail -3
for T in "" 2000000 600000 200000; do echo "THREAD_MIN=$T"; BEAST_IR_THREAD_MIN=$T timeout 300 python scripts/ir_time.py headline widened256_k40c 2>&1 | grep -o "IR count.*same stats: [A-Za-z]*"; done
