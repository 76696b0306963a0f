# loader with a CTA-level box reduction: parity + the launch list (loader time)
mkdir -p gpurun_out/r2w
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -q -x > gpurun_out/r2w/pytest.txt 2>&1; tail -2 gpurun_out/r2w/pytest.txt
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "1m or 4m_lattice or validate" > gpurun_out/r2w/pytest_fs.txt 2>&1; tail -2 gpurun_out/r2w/pytest_fs.txt
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2w/launches_sdh_uniform_1m.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/r2w/launches.log 2>&1
grep soa_loader gpurun_out/r2w/launches_sdh_uniform_1m.csv | head -6
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2w/launches_sdh_uniform_4m.csv \
  python bench.py --workload sdh_uniform_4m --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r2w/launches4m.log 2>&1
grep soa_loader gpurun_out/r2w/launches_sdh_uniform_4m.csv | head -6
