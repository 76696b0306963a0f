# SDH 1M: slot order / two-phase grouping A/B (mq1 anchor-major, mq2 two phases over 16 slots, mq3 over 4)
mkdir -p gpurun_out/r2y
bash tools/ab_run.sh sdh_uniform_1m 10 main mq1 mq2 mq3 main mq1 mq2 mq3 > gpurun_out/r2y/ab.txt 2>&1; cut -c1-90 gpurun_out/r2y/ab.txt
