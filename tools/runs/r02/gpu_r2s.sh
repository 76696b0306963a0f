# fused combine in the pair kernel's tail: fused-combine + parity GPU tests, bench lines, new peaks
mkdir -p gpurun_out/r2s
timeout 900 python -m pytest tests/test_gpu_fused.py tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/r2s/pytest.txt 2>&1
tail -3 gpurun_out/r2s/pytest.txt
python bench.py --no-cpu-baseline > gpurun_out/r2s/bench_default.json 2>&1; tail -c 400 gpurun_out/r2s/bench_default.json
python bench.py --no-cpu-baseline --workload pcf_clustered_4m --steps 3 > gpurun_out/r2s/bench_pcf.json 2>&1; tail -c 300 gpurun_out/r2s/bench_pcf.json
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/peaks tools/peaks.cu && /tmp/peaks > gpurun_out/r2s/peaks.json 2>&1; cat gpurun_out/r2s/peaks.json
