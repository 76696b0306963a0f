for b in 32 64 128 256; do
  echo band $b; TBS_HD_BAND=$b bash tools/ab_run.sh pairmatrix_hd_64k_d512 5 main
done
for b in 32 256; do
  echo band $b; TBS_HD_BAND=$b bash tools/ab_run.sh pairmatrix_hd_64k_d64 5 main
done
