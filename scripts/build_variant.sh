#!/bin/bash
# usage: scripts/build_variant.sh NAME [-DFLAG=..]... — in-tree variant build variants/NAME.so (same sources, extra defines)
NAME=$1; shift
cd "$(dirname "$0")/.." || exit 1
mkdir -p variants
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared \
  -diag-suppress 128 "$@" -I include -o variants/$NAME.so paper_conf_ipps_luszczekgkdd16_b200/csrc/beast.cu \
  paper_conf_ipps_luszczekgkdd16_b200/csrc/beast_ir.cu -ldl 2>&1 | grep -iE " error" ; echo "built variants/$NAME.so"
