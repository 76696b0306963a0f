set -x
timeout 300 python -m pytest tests -q -m gpu -x -k "hd" 2>&1 | tail -5
for wl in pairmatrix_hd_64k_d512; do
  timeout 120 python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-250
done
TBS_HD_1SM=0 timeout 120 python bench.py --workload pairmatrix_hd_64k_d64 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-250
