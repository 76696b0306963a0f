set -x
timeout 300 python -m pytest tests -q -m gpu -x -k "hd_ast" 2>&1 | tail -3
for v in r3s2 r4s1; do
  TBS_LIB_VARIANT=build/ab/libtbs_$v.so TBS_HD_AST=1 timeout 200 python bench.py --workload pairmatrix_hd_64k_d512 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v', round(d['value'],1), 'kms', round(r['kernel_ms_avg'],3))"
done
TBS_HD_AST=0 timeout 200 python bench.py --workload pairmatrix_hd_64k_d512 --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('hd2', round(d['value'],1), 'kms', round(r['kernel_ms_avg'],3))"
