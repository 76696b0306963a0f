set -x
mkdir -p gpurun_out/r2f
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -x -q > gpurun_out/r2f/pytest.txt 2>&1
tail -2 gpurun_out/r2f/pytest.txt
python tools/c1_probe.py > gpurun_out/r2f/c1_probe.jsonl 2>&1
for r in 4 3 2; do TBS_LOG2R=$r python tools/c1_probe.py >> gpurun_out/r2f/c1_probe.jsonl 2>&1; done
B="timeout 600 python bench.py --no-cpu-baseline"
$B --workload sdh_uniform_4k --steps 50 > gpurun_out/r2f/c1_graph.json 2>&1
timeout 300 python tools/c1_e2e.py > gpurun_out/r2f/c1_e2e.json 2>&1
$B > gpurun_out/r2f/bench_1m.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 20 -c 1 -o gpurun_out/r2f/prof_c1 python tools/c1_probe.py > gpurun_out/r2f/ncu_c1.log 2>&1
