# round 2: full GPU suite + sanitizers at HEAD, C1 small path (graph, static items, e2e host cost),
# Fig. 7 ablation (hoisted LB tail), FP32 pipe-mix peaks, default bench lines
set -x
mkdir -p gpurun_out/r2d
timeout 3600 python -m pytest tests -m gpu -q > gpurun_out/r2d/pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2d/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2d/smoke.txt 2>&1
./tools/peaks > gpurun_out/r2d/peaks.json 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ablate_intra tools/ablate_intra.cu && /tmp/ablate_intra > gpurun_out/r2d/ablate_intra.jsonl 2>&1
B="timeout 600 python bench.py --no-cpu-baseline"
$B --workload sdh_uniform_4k --steps 50 > gpurun_out/r2d/c1_graph.json 2>&1
$B --workload sdh_uniform_4k --steps 50 --graph off > gpurun_out/r2d/c1_nograph.json 2>&1
timeout 300 python tools/c1_e2e.py > gpurun_out/r2d/c1_e2e.json 2>&1
python bench.py > gpurun_out/r2d/bench_sdh_uniform_1m.json 2>&1
$B --workload sdh_uniform_2m_16k --steps 3 > gpurun_out/r2d/bench_sdh_uniform_2m_16k.json 2>&1
mkdir -p gpurun_out/r2d/san
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/sanitize_driver.py 2500 \
    > gpurun_out/r2d/san/sanitize_$tool.log 2>&1
  echo "$tool exit $?"
done
