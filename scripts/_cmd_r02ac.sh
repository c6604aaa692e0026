bash scripts/ab2.sh "headline b200_S" variants/noF.so
bash scripts/ab2.sh "headline" variants/noF.so
