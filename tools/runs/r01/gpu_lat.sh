set -x
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -4
timeout 300 python bench.py --workload sdh_lattice_4m --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_sdh_lattice_4m.json 2>&1; tail -1 gpurun_out/bench_sdh_lattice_4m.json
