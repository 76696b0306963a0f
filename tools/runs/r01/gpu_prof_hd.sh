wl=${1:-pairmatrix_hd_64k_d512}; tag=${2:-hd512}
ncu --set full --clock-control none --import-source on -k regex:hd_pairmatrix -s 2 -c 1 -o gpurun_out/prof_$tag \
  python bench.py --workload $wl --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_$tag.log 2>&1
tail -2 gpurun_out/ncu_$tag.log
