# round 2, first GPU call: peaks, HEAD bench lines with the NVML clock sampler, C4 R/occupancy
# experiments, ncu captures of the SDH 1M and C4 pair kernels at HEAD.
set -x
mkdir -p gpurun_out/r2a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r2a/smi.txt
./tools/peaks > gpurun_out/r2a/peaks.json 2> gpurun_out/r2a/peaks.err
B="timeout 600 python bench.py --no-cpu-baseline"
python bench.py > gpurun_out/r2a/bench_sdh_uniform_1m.json 2> gpurun_out/r2a/bench_sdh_uniform_1m.err
for wl in sdh_uniform_2m_16k pairmatrix_64k pairmatrix_hd_64k_d64 pairmatrix_hd_64k_d512 kde_uniform_1m sdh_uniform_4k knn_uniform_1m_k8 pcf_clustered_4m; do
  $B --workload $wl > gpurun_out/r2a/bench_$wl.json 2> gpurun_out/r2a/bench_$wl.err
done
TBS_LOG2R=0 $B --workload sdh_uniform_2m_16k > gpurun_out/r2a/c4_r1.json 2>&1
TBS_LOG2R=0 TBS_OCC=1 $B --workload sdh_uniform_2m_16k > gpurun_out/r2a/c4_r1_occ1.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o gpurun_out/r2a/prof_sdh1m \
  python bench.py --workload sdh_uniform_1m --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r2a/ncu_sdh1m.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o gpurun_out/r2a/prof_c4 \
  python bench.py --workload sdh_uniform_2m_16k --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r2a/ncu_c4.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2a/launches_sdh1m.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/r2a/launches.log 2>&1
ls -la gpurun_out/r2a
