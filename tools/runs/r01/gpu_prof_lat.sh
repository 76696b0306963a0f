set -x
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_sdh_uniform_1m.json 2> gpurun_out/bench_default.err; tail -1 gpurun_out/bench_sdh_uniform_1m.json | cut -c1-300
python bench.py --workload sdh_lattice_4m --steps 3 --warmup 3 > gpurun_out/bench_sdh_lattice_4m.json 2>&1; tail -1 gpurun_out/bench_sdh_lattice_4m.json | cut -c1-300
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_sdh_lattice_4m.csv python bench.py --workload sdh_lattice_4m --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 6 -c 1 -o gpurun_out/prof_lat4m_bias python bench.py --workload sdh_lattice_4m --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_lat.log 2>&1
tail -2 gpurun_out/ncu_lat.log
