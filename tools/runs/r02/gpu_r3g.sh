# bounds-checked build (TBS_BOUNDS_CHECK: every histogram increment address checked, trap on a miss)
# over the GPU parity and fused-combine suites, the entry-point driver and full-size workloads
mkdir -p gpurun_out/r3g
export TBS_LIB_VARIANT=build/ab/libtbs_bounds.so
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py -m gpu -q > gpurun_out/r3g/pytest.txt 2>&1; tail -2 gpurun_out/r3g/pytest.txt
timeout 600 python tools/sanitize_driver.py 2500 > gpurun_out/r3g/driver_2500.txt 2>&1; tail -1 gpurun_out/r3g/driver_2500.txt
timeout 600 python tools/sanitize_driver.py 40000 > gpurun_out/r3g/driver_40000.txt 2>&1; tail -1 gpurun_out/r3g/driver_40000.txt
for wl in sdh_uniform_4k sdh_uniform_1m sdh_uniform_2m_16k sdh_lattice_4m pcf_clustered_4m kde_uniform_1m; do
  timeout 600 python bench.py --no-cpu-baseline --workload $wl --steps 1 --warmup 3 > gpurun_out/r3g/bench_$wl.json 2>&1; echo "$wl exit $? $(tail -c 200 gpurun_out/r3g/bench_$wl.json | tr -d '\n' | cut -c1-120)"
done
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -k "16k or lattice or max_n" > gpurun_out/r3g/pytest_fs.txt 2>&1; tail -2 gpurun_out/r3g/pytest_fs.txt
