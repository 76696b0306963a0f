# tensor-core pair matrix: operand ring depth vs epilogue staging buffers (A/B builds), parity first
mkdir -p gpurun_out/r2r
for v in s24 s15 s33 l33; do
  TBS_LIB_VARIANT=build/ab/libtbs_$v.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "pairmatrix_hd" > gpurun_out/r2r/pytest_$v.txt 2>&1
  echo "$v parity: $(tail -1 gpurun_out/r2r/pytest_$v.txt)"
done
timeout 600 bash tools/ab_run.sh pairmatrix_hd_64k_d64 10 main s24 s15 s33 main > gpurun_out/r2r/ab_d64.txt 2>&1
timeout 600 bash tools/ab_run.sh pairmatrix_hd_64k_d512 10 main l33 main > gpurun_out/r2r/ab_d512.txt 2>&1
cut -c1-100 gpurun_out/r2r/ab_d64.txt gpurun_out/r2r/ab_d512.txt
