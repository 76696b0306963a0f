# lattice one-sided variant without the 4^j s < 2^24 condition: exact-lattice GPU tests (all sizes) + C4 lattice bench line
mkdir -p gpurun_out/r3z
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_fused.py -m gpu -q -k "lattice" > gpurun_out/r3z/pytest.txt 2>&1; tail -2 gpurun_out/r3z/pytest.txt
python bench.py --no-cpu-baseline --workload sdh_lattice_2m_16k --steps 3 > gpurun_out/r3z/bench_sdh_lattice_2m_16k.json 2> gpurun_out/r3z/err.txt; tail -c 700 gpurun_out/r3z/bench_sdh_lattice_2m_16k.json
python bench.py --no-cpu-baseline --workload sdh_lattice_4m --steps 3 > gpurun_out/r3z/bench_sdh_lattice_4m.json 2>> gpurun_out/r3z/err.txt; tail -c 300 gpurun_out/r3z/bench_sdh_lattice_4m.json
