# round 2: GPU parity (RDF rework, validation, sqrt bound) + FMA-pipe sqrt A/B (TBS_SW_SQRT)
set -x
mkdir -p gpurun_out/r2b
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/r2b/pytest_parity.txt 2>&1
tail -3 gpurun_out/r2b/pytest_parity.txt
for v in sw1 sw1b sw2 sw2b; do
  TBS_LIB_VARIANT=build/ab/libtbs_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "uniform_ragged or main_config" > gpurun_out/r2b/pytest_$v.txt 2>&1
  tail -1 gpurun_out/r2b/pytest_$v.txt
done
for rep in 1 2; do
for v in base sw1 sw1b sw2 sw2b; do
  if [ $v = base ]; then L=paper_conf_icpp_pitaksirianannt16_b200/libtbs.so; else L=build/ab/libtbs_$v.so; fi
  TBS_LIB_VARIANT=$L timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/r2b/bench_${v}_$rep.json 2>&1
  TBS_LIB_VARIANT=$L timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload sdh_uniform_4m > gpurun_out/r2b/bench4m_${v}_$rep.json 2>&1
done
done
for v in sw1 sw2; do
ncu --set full --clock-control none -k regex:pair_kernel -s 3 -c 1 -o gpurun_out/r2b/prof_$v \
  env TBS_LIB_VARIANT=build/ab/libtbs_$v.so python bench.py --workload sdh_uniform_1m --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r2b/ncu_$v.log 2>&1
done
