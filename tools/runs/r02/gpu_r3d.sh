# ncu of the windowed pair kernel at 2M / 16K
mkdir -p gpurun_out/r3d
TBS_WIN=1 ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o /tmp/prof_win \
  python bench.py --workload sdh_uniform_2m_16k --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r3d/ncu.log 2>&1
python tools/ncu_summary.py /tmp/prof_win.ncu-rep > gpurun_out/r3d/ncu_summary_win.txt 2>&1
ncu -i /tmp/prof_win.ncu-rep --page details > gpurun_out/r3d/ncu_details_win.txt 2>&1
ncu -i /tmp/prof_win.ncu-rep --page source --csv > gpurun_out/r3d/ncu_source_win.csv 2>&1
ls -la gpurun_out/r3d; head -30 gpurun_out/r3d/ncu_summary_win.txt
