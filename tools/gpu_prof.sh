# usage: bash tools/gpu_prof.sh WORKLOAD TAG   -> gpurun_out/prof_<TAG>.ncu-rep (one pair-kernel launch, --set full)
wl=$1; tag=$2
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o gpurun_out/prof_$tag \
  python bench.py --workload $wl --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_$tag.log 2>&1
tail -2 gpurun_out/ncu_$tag.log
