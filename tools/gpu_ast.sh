# A-stationary hd kernel: parity (hd tests) + A/B against the hd2 kernel at 64K x 512.
set -x
timeout 400 python -m pytest tests -q -m gpu -x -k "hd" 2>&1 | tail -5
for ast in 0 1; do
  TBS_HD_AST=$ast timeout 200 python bench.py --workload pairmatrix_hd_64k_d512 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('ast=$ast', round(d['value'],1), d['unit'], 'kms', round(r['kernel_ms_avg'],3), r.get('tensor_view'), d['clocks'])"
done
