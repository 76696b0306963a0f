# C1 (N = 4096) line with enough steps for the 5 ms NVML clock sampler to see the timed region
mkdir -p gpurun_out/r4c
python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 3000 > gpurun_out/r4c/bench_sdh_uniform_4k.json 2>&1; tail -c 400 gpurun_out/r4c/bench_sdh_uniform_4k.json
