# round 2: full GPU suite at HEAD, Fig. 9 / Fig. 7 ablations, C1 small-path variants
set -x
mkdir -p gpurun_out/r2c
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ablate_intra tools/ablate_intra.cu
/tmp/ablate_intra > gpurun_out/r2c/ablate_intra.jsonl 2> gpurun_out/r2c/ablate_intra.err
B="timeout 600 python bench.py --no-cpu-baseline"
for v in base pp1 pp2; do
  if [ $v = base ]; then L=paper_conf_icpp_pitaksirianannt16_b200/libtbs.so; else L=build/ab/libtbs_$v.so; fi
  TBS_LIB_VARIANT=$L $B > gpurun_out/r2c/fig9_${v}_1m.json 2>&1
  TBS_LIB_VARIANT=$L $B --workload sdh_uniform_2m_16k --steps 3 > gpurun_out/r2c/fig9_${v}_16k.json 2>&1
done
for v in base st32 st128 st256; do
  if [ $v = base ]; then L=paper_conf_icpp_pitaksirianannt16_b200/libtbs.so; else L=build/ab/libtbs_$v.so; fi
  TBS_LIB_VARIANT=$L $B --workload sdh_uniform_4k --steps 50 > gpurun_out/r2c/c1_${v}.json 2>&1
done
timeout 3000 python -m pytest tests -m gpu -x -q > gpurun_out/r2c/pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2c/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2c/smoke.txt 2>&1
