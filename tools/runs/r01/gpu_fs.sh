timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -m gpu -x -k "d512 or kde" 2>&1 | tail -3
timeout 300 python bench.py --workload sdh_uniform_2m_16k --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline'])"
