# lane-private trash words vs one trash word per replica (HEAD build): bucket passes, C4, CTA mode; atomics microbenchmarks
mkdir -p gpurun_out/r2t
./tools/peaks > gpurun_out/r2t/peaks.json 2>&1
python -c "
import json; d=json.load(open('gpurun_out/r2t/peaks.json'))
for k in sorted(d):
    if 'atoms' in k or k in ('f2i','shfl_idx_lanes'): print(k, d[k])
"
for v in head main; do
  lib=""; [ $v = head ] && lib=build/ab/libtbs_head.so
  TBS_LIB_VARIANT=$lib timeout 600 python tools/ab_nb.py 256 256:cta 16384 49152 65536 131072 16384:passes > gpurun_out/r2t/ab_nb_$v.jsonl 2>&1
  cat gpurun_out/r2t/ab_nb_$v.jsonl
done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -q -x -k "passes or hist_modes or lattice_replication or fanout or 16k" > gpurun_out/r2t/pytest.txt 2>&1; tail -2 gpurun_out/r2t/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "16k" > gpurun_out/r2t/pytest_fs.txt 2>&1; tail -2 gpurun_out/r2t/pytest_fs.txt
