# partner-major slot order for bucket-range passes: nb sweep points around the passes
mkdir -p gpurun_out/r3i
timeout 600 python tools/ab_nb.py 256 4096 16384 49152 65536 98304 131072 16384:passes > gpurun_out/r3i/ab_nb.jsonl 2>&1; cat gpurun_out/r3i/ab_nb.jsonl
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "passes or hist_modes or replication" > gpurun_out/r3i/pytest.txt 2>&1; tail -1 gpurun_out/r3i/pytest.txt
