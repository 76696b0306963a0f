set -x
mkdir -p gpurun_out/r2m
timeout 300 python tools/c1_e2e.py > gpurun_out/r2m/c1_e2e.json 2>&1
timeout 300 python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 50 > gpurun_out/r2m/c1_graph.json 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -x -q > gpurun_out/r2m/pytest.txt 2>&1
tail -2 gpurun_out/r2m/pytest.txt
