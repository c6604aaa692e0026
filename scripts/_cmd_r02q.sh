timeout 900 python -m pytest -x -q tests/test_gpu_ir.py 2>&1 | tail -2
BEAST_IR_TRACE=1 python scripts/ir_time.py headline b200_D 2>&1 | grep -v "^ir level" ; BEAST_IR_TRACE=1 python scripts/ir_time.py headline 2>&1 | tail -16
BEAST_IR_MATERIALIZE_MAX=268435456 python scripts/ir_time.py headline b200_D 2>&1 | tail -2
