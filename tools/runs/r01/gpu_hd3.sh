timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "hd" 2>&1 | tail -2
for wl in pairmatrix_hd_64k_d64 pairmatrix_hd_64k_d512; do
  timeout 120 python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$wl', d['value'], d['roofline']['kernel_ms_avg'], d['roofline']['frac'])"
done
