# one-sided lattice variant at large x (pinning test)
mkdir -p gpurun_out/r4a
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "one_sided_large_x or lattice" > gpurun_out/r4a/pytest.txt 2>&1; tail -3 gpurun_out/r4a/pytest.txt
