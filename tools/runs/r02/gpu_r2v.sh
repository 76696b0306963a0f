# small-problem (N = 4096) fused-kernel tile shape A/B: host-buffer call and graph-replayed step
mkdir -p gpurun_out/r2v
for v in main stp64 stp256 ska4 main; do
  lib=""; [ $v != main ] && lib=build/ab/libtbs_$v.so
  echo "$v $(TBS_LIB_VARIANT=$lib timeout 300 python tools/c1_e2e.py 2>&1 | tail -1)"
  TBS_LIB_VARIANT=$lib timeout 300 python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 200 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v step_us', round(d['ms_per_step']*1e3,2), 'e2e', round(d['e2e']['value'],1))"
done > gpurun_out/r2v/ab_small.txt 2>&1
cat gpurun_out/r2v/ab_small.txt
