# write rate by tile raster (round-robin vs contiguous ranges) + hd pair-matrix raster bands at d = 64 / 512
set -x
mkdir -p gpurun_out/r2p
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/write_pattern tools/write_pattern.cu
timeout 300 /tmp/write_pattern > gpurun_out/r2p/write_pattern.jsonl 2>&1
cat gpurun_out/r2p/write_pattern.jsonl
for b in 0 1 2 4 -1; do
  TBS_HD_BAND=$b timeout 300 python bench.py --workload pairmatrix_hd_64k_d64 --steps 10 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('d64 band $b', d['ms_per_step'], d['value'], d['roofline']['frac'], d['clocks']['sm_mhz'])"
done
for b in 1 2 4 32; do
  TBS_HD_BAND=$b timeout 300 python bench.py --workload pairmatrix_hd_64k_d512 --steps 10 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('d512 band $b', d['ms_per_step'], d['value'], d['roofline']['frac'], d['clocks']['sm_mhz'])"
done
