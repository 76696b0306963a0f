# hd epilogue: TMA-only stores vs LSU/TMA mixes (TBS_HD_LSU_MASK): parity + A/B at d = 64 and 512.
set -x
for v in lsuA lsuF; do
  TBS_LIB_VARIANT=build/ab/libtbs_$v.so timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "hd" 2>&1 | tail -2
done
for wl in pairmatrix_hd_64k_d64 pairmatrix_hd_64k_d512; do
  for v in main lsu8 lsuA lsu5 lsuF; do
    if [ "$v" = main ]; then lib=""; else lib=build/ab/libtbs_$v.so; fi
    TBS_LIB_VARIANT=$lib timeout 200 python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$wl', '$v', round(d['value'],1), 'kms', round(r['kernel_ms_avg'],3))"
  done
done
