set -x
timeout 600 python -m pytest tests -q -m gpu -x -k "hd" 2>&1 | tail -3
for wl in pairmatrix_hd_64k_d64 pairmatrix_hd_64k_d512; do
  timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$wl.json 2>&1; tail -1 gpurun_out/bench_$wl.json
done
bash tools/runs/r01/gpu_prof_hd.sh pairmatrix_hd_64k_d512 hd512b
