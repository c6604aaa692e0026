# tile schedule variants (guide factor, smallest tile, 1024-job tiles)
mkdir -p gpurun_out
bash scripts/ab2.sh "headline b200_S" variants/g1.so variants/min128.so variants/g1min256.so variants/tj1024.so
