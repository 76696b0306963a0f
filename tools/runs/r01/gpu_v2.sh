set -x
timeout 600 python -m pytest tests/test_gpu_fused.py -q -x 2>&1 | tail -3
timeout 300 python bench.py --workload sdh_lattice_4m --steps 3 --warmup 3 > gpurun_out/bench_sdh_lattice_4m.json 2>&1; tail -1 gpurun_out/bench_sdh_lattice_4m.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e'], d['config']['combine'])"
