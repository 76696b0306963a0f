# One GPU session: parity suites, every bench workload, the default bench line, ncu launch list.
set -x
python -m pytest tests/test_gpu_parity.py -q -m gpu -x 2>&1 | tail -2
python bench.py --steps 10 --warmup 3 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; cat gpurun_out/bench_default.json
for wl in sdh_uniform_4k sdh_clustered_1m sdh_uniform_4m sdh_uniform_2m_16k sdh_lattice_4m pcf_clustered_4m pairmatrix_64k; do
  python bench.py --workload $wl --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$wl.json 2>&1; tail -1 gpurun_out/bench_$wl.json
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
