# small fused kernel: histogram replicas (R = 32 main, 16, 8, 4): graph step and host-buffer call at N = 4096
mkdir -p gpurun_out/r3t
for v in main sr4 sr3 sr2 main; do
  lib=""; [ $v != main ] && lib=build/ab/libtbs_$v.so
  TBS_LIB_VARIANT=$lib timeout 300 python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 500 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v step_us', round(d['ms_per_step']*1e3,2), 'e2e', round(d['e2e']['value'],1))"
  echo "$v $(TBS_LIB_VARIANT=$lib timeout 300 python tools/c1_e2e.py 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('host_us', round(d['us_host_entry_pinned_in'],2))")"
done | tee gpurun_out/r3t/ab.txt
TBS_LIB_VARIANT=build/ab/libtbs_sr3.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "host or small or config1 or uniform_ragged" > gpurun_out/r3t/pytest_sr3.txt 2>&1; tail -1 gpurun_out/r3t/pytest_sr3.txt
