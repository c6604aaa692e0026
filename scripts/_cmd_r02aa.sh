bash scripts/ab2.sh "headline b200_S" variants/un2.so variants/un3.so variants/un8.so variants/cu2.so variants/fc1.so variants/fc2.so variants/fc4.so
