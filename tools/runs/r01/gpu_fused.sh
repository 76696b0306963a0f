set -x
timeout 600 python -m pytest tests/test_gpu_fused.py -q -x 2>&1 | tail -15
timeout 1500 python -m pytest tests -q -m gpu -x 2>&1 | tail -3
bash tools/ab_run.sh sdh_uniform_1m 5 main
bash tools/ab_run.sh pcf_clustered_4m 2 main
