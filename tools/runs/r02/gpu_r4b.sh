# final verification at HEAD (one-sided lattice admission): full GPU suite, smoke, default and C1 bench lines, c1_e2e
mkdir -p gpurun_out/r4b
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r4b/smi.txt
timeout 3000 python -m pytest tests -m gpu -q > gpurun_out/r4b/pytest_gpu.txt 2>&1; tail -2 gpurun_out/r4b/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r4b/smoke.txt 2>&1; cat gpurun_out/r4b/smoke.txt
python bench.py > gpurun_out/r4b/bench_default.json 2> gpurun_out/r4b/bench_default.err; tail -c 300 gpurun_out/r4b/bench_default.json
python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 3000 > gpurun_out/r4b/bench_sdh_uniform_4k.json 2>&1; tail -c 300 gpurun_out/r4b/bench_sdh_uniform_4k.json
timeout 300 python tools/c1_e2e.py > gpurun_out/r4b/c1_e2e.json 2>&1; cat gpurun_out/r4b/c1_e2e.json
