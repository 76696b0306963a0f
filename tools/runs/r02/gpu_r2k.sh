set -x
mkdir -p gpurun_out/r2k
TBS_HOST_TRACE=1 timeout 300 python tools/c1_e2e.py > gpurun_out/r2k/c1_e2e.json 2> gpurun_out/r2k/c1_e2e.err
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -x -q > gpurun_out/r2k/pytest.txt 2>&1
tail -2 gpurun_out/r2k/pytest.txt
