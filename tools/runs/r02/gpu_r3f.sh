# SDH 1M config A/B with the anchor-major slot order (TP 512/2048, KA 4 at 4 CTAs/SM, unroll 2)
mkdir -p gpurun_out/r3f
bash tools/ab_run.sh sdh_uniform_1m 10 main am_tp512 am_tp2k am_ka4m4 am_pu2 main > gpurun_out/r3f/ab.txt 2>&1
cut -c1-95 gpurun_out/r3f/ab.txt
