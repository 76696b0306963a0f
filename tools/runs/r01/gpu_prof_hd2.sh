ncu --set full --clock-control none --import-source on -k regex:hd_pair -s 2 -c 1 -o gpurun_out/prof_hd512c \
  python bench.py --workload pairmatrix_hd_64k_d512 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_hd512c.log 2>&1
tail -2 gpurun_out/ncu_hd512c.log
