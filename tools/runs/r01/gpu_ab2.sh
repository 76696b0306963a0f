timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "hd" 2>&1 | tail -2
bash tools/ab_run.sh pairmatrix_hd_64k_d64 5 main nostore
bash tools/ab_run.sh pairmatrix_hd_64k_d512 5 main nostore
