# configs[3] in exact-lattice mode: N = 128^3, 16384 buckets, w = 2^-6 (one-sided fix-up variant, 2 replicas)
mkdir -p gpurun_out/r3y
python bench.py --no-cpu-baseline --workload sdh_lattice_2m_16k --steps 3 > gpurun_out/r3y/bench_sdh_lattice_2m_16k.json 2> gpurun_out/r3y/err.txt; tail -c 600 gpurun_out/r3y/bench_sdh_lattice_2m_16k.json; tail -3 gpurun_out/r3y/err.txt
