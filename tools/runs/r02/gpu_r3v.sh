# per-device small scratch: host/small GPU tests + c1 e2e
mkdir -p gpurun_out/r3v
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -q > gpurun_out/r3v/pytest.txt 2>&1; tail -1 gpurun_out/r3v/pytest.txt
timeout 300 python tools/c1_e2e.py > gpurun_out/r3v/c1_e2e.json 2>&1; cat gpurun_out/r3v/c1_e2e.json
