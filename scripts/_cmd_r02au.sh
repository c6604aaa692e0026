mkdir -p gpurun_out
timeout 600 python scripts/ir_sweep.py headline BEAST_IR_SHORT_TRIP 0 8 64
timeout 300 python scripts/ir_sweep.py b200_D BEAST_IR_SHORT_TRIP 0 8
timeout 900 python -m pytest -x -q tests/test_gpu_ir.py tests/test_ir_compile.py 2>&1 | tail -2
