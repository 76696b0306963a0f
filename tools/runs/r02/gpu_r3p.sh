# kernel density on its own config (3 CTAs/SM): KDE GPU tests + bench line
mkdir -p gpurun_out/r3p
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -k "kde" > gpurun_out/r3p/pytest.txt 2>&1; tail -1 gpurun_out/r3p/pytest.txt
python bench.py --no-cpu-baseline --workload kde_uniform_1m --steps 10 > gpurun_out/r3p/bench_kde_uniform_1m.json 2>&1; tail -c 300 gpurun_out/r3p/bench_kde_uniform_1m.json
