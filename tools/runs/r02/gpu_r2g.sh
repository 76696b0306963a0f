set -x
mkdir -p gpurun_out/r2g
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -x -q > gpurun_out/r2g/pytest.txt 2>&1
tail -2 gpurun_out/r2g/pytest.txt
for v in base st64 st32; do
  if [ $v = base ]; then L=paper_conf_icpp_pitaksirianannt16_b200/libtbs.so; else L=build/ab/libtbs_$v.so; fi
  TBS_LIB_VARIANT=$L python tools/c1_probe.py | sed "s/^/$v /" >> gpurun_out/r2g/c1_probe.txt 2>&1
  TBS_LIB_VARIANT=$L timeout 300 python bench.py --no-cpu-baseline --workload sdh_uniform_4k --steps 50 > gpurun_out/r2g/c1_graph_$v.json 2>&1
  TBS_LIB_VARIANT=$L timeout 300 python tools/c1_e2e.py > gpurun_out/r2g/c1_e2e_$v.json 2>&1
done
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/r2g/bench_1m.json 2>&1
