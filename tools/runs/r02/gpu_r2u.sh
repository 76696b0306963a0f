# verification at HEAD after the fused-tail combine: full GPU suite, smoke, default bench line
mkdir -p gpurun_out/r2u
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r2u/smi.txt
timeout 3000 python -m pytest tests -m gpu -q > gpurun_out/r2u/pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2u/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2u/smoke.txt 2>&1; cat gpurun_out/r2u/smoke.txt
python bench.py > gpurun_out/r2u/bench_default.json 2> gpurun_out/r2u/bench_default.err; tail -c 600 gpurun_out/r2u/bench_default.json
