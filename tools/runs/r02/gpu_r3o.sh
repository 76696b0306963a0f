# 2PCF / KDE config A/B: 3 CTAs/SM (80 registers) or KA 4 at 4 CTAs/SM vs the product (KA 8, 2 CTAs/SM)
mkdir -p gpurun_out/r3o
bash tools/ab_run.sh kde_uniform_1m 10 main pcfm3 pcfka4m4 main > gpurun_out/r3o/ab.txt 2>&1
bash tools/ab_run.sh pcf_clustered_4m 3 main pcfm3 pcfka4m4 >> gpurun_out/r3o/ab.txt 2>&1
cut -c1-95 gpurun_out/r3o/ab.txt
