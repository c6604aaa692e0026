# IR engine per-level trace, headline
mkdir -p gpurun_out
BEAST_IR_TRACE=1 timeout 600 python scripts/ir_time.py headline 2>&1 | tail -30
