BEAST_IR_TRACE=1 python scripts/ir_time.py headline headline 2>&1 | tail -34
bash scripts/ab2.sh "headline b200_S" variants/ki14.so variants/ki16.so
