set -x
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
cat gpurun_out/bench_default.json; tail -5 gpurun_out/bench_default.err
python bench.py --workload pcf_clustered_4m --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_pcf.json 2>&1; cat gpurun_out/bench_pcf.json | tail -3
python bench.py --workload sdh_uniform_2m_16k --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_16k.json 2>&1; tail -3 gpurun_out/bench_16k.json
python bench.py --workload pairmatrix_64k --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_pm.json 2>&1; tail -3 gpurun_out/bench_pm.json
python bench.py --workload sdh_lattice_4m --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_lat.json 2>&1; tail -3 gpurun_out/bench_lat.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o gpurun_out/prof_sdh_r01 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
