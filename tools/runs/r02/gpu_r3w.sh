# NEXT-1 bench line: RDF N = 1M (SDH with nb + 1 buckets + the device normalisation)
mkdir -p gpurun_out/r3w
python bench.py --no-cpu-baseline --workload rdf_uniform_1m --steps 10 > gpurun_out/r3w/bench_rdf_uniform_1m.json 2> gpurun_out/r3w/err.txt; tail -c 700 gpurun_out/r3w/bench_rdf_uniform_1m.json; tail -3 gpurun_out/r3w/err.txt
