timeout 900 python -m pytest -x -q tests/test_gpu_ir.py 2>&1 | tail -2
BEAST_IR_TRACE=1 python scripts/ir_time.py headline 2>&1 | tail -16
python scripts/ir_time.py headline b200_D b200_S 2>&1 | tail -3
