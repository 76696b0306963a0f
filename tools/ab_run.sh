# usage: bash tools/ab_run.sh WORKLOAD STEPS variant...   (variants in build/ab/libtbs_<v>.so; "main" = in-tree lib)
wl=$1; steps=$2; shift 2
for v in "$@"; do
  if [ "$v" = main ]; then lib=""; else lib=build/ab/libtbs_$v.so; fi
  TBS_LIB_VARIANT=$lib python bench.py --workload $wl --steps $steps --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', '$wl', round(d['value'],1), d['unit'], 'frac', round(d['roofline']['frac'],4), 'kms', round(d['roofline']['kernel_ms_avg'],2), d['clocks'])"
done
