# small host-buffer path: programmatic dependent launch of the fused kernel after the copy kernel (default) vs none
mkdir -p gpurun_out/r3l
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "host or small or graph or kde or rdf or knn_host" > gpurun_out/r3l/pytest.txt 2>&1; tail -1 gpurun_out/r3l/pytest.txt
for v in 1 0 1 0; do
  echo "pdl=$v $(TBS_SMALL_PDL=$v TBS_HOST_TRACE=1 timeout 300 python tools/c1_e2e.py 2>gpurun_out/r3l/trace_$v.err | tail -1 | cut -c1-330)"; tail -1 gpurun_out/r3l/trace_$v.err
done
timeout 300 python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 200 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench 4k step_us', round(d['ms_per_step']*1e3,2), 'e2e', round(d['e2e']['value'],1))"
