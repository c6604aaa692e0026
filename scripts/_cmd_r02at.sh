mkdir -p gpurun_out
timeout 600 python scripts/ir_sweep.py headline BEAST_IR_THREAD_MIN - 20000000 4000000 2000000 1000000 500000 200000
timeout 300 python scripts/ir_sweep.py b200_D BEAST_IR_THREAD_MIN - 2000000 1000000 500000
