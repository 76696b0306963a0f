# SDH 1M: order of the (partner, anchor-pair) slots in a group (partner-major main vs anchor-major mq1)
mkdir -p gpurun_out/r2x
bash tools/ab_run.sh sdh_uniform_1m 10 main mq1 main mq1 > gpurun_out/r2x/ab.txt 2>&1; cut -c1-90 gpurun_out/r2x/ab.txt
