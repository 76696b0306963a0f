# write rate: persistent tile CTAs vs the Type-III kernel's non-persistent 2-D grid vs memset
mkdir -p gpurun_out/r2q
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/write_pattern tools/write_pattern.cu
timeout 300 /tmp/write_pattern > gpurun_out/r2q/write_pattern.jsonl 2>&1
cat gpurun_out/r2q/write_pattern.jsonl
