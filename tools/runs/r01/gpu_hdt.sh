timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "hd" 2>&1 | tail -3
TBS_HD_1SM=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "hd" 2>&1 | tail -3
