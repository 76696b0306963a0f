set -x
mkdir -p gpurun_out/r2i
ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg --clock-control none --csv --log-file gpurun_out/r2i/c1_launches.csv python tools/c1_probe.py > gpurun_out/r2i/c1.log 2>&1
ncu --set full --clock-control none -k regex:soa_loader -s 20 -c 1 -o gpurun_out/r2i/prof_loader python tools/c1_probe.py > gpurun_out/r2i/ncu_loader.log 2>&1
