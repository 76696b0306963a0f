# HBM write rate by tile shape (tools/write_pattern.cu) + KDE 1M: HEAD vs the 67bfb35 build (same hot-loop SASS)
set -x
mkdir -p gpurun_out/r2o
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/write_pattern tools/write_pattern.cu
timeout 300 /tmp/write_pattern > gpurun_out/r2o/write_pattern.jsonl 2>&1
cat gpurun_out/r2o/write_pattern.jsonl
timeout 600 bash tools/ab_run.sh kde_uniform_1m 10 main old67 main > gpurun_out/r2o/ab_kde.txt 2>&1
cat gpurun_out/r2o/ab_kde.txt
