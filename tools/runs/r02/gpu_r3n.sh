# ncu source view of the small fused kernel (N = 4096, configs[0])
mkdir -p gpurun_out/r3n
ncu --set full --clock-control none --import-source on -k regex:pair_kernel_small -s 20 -c 1 -o /tmp/prof_small python tools/c1_probe.py > gpurun_out/r3n/ncu.log 2>&1
python tools/ncu_summary.py /tmp/prof_small.ncu-rep > gpurun_out/r3n/summary.txt 2>&1
ncu -i /tmp/prof_small.ncu-rep --page source --csv > gpurun_out/r3n/source.csv 2>&1
head -5 gpurun_out/r3n/summary.txt; ls -la gpurun_out/r3n
