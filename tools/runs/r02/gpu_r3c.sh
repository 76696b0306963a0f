# windowed large-nb SDH: parity, then the C4 A/B (TBS_WIN=0 plain, =1 windowed)
mkdir -p gpurun_out/r3c
timeout 900 python -m pytest tests/test_gpu_window.py -m gpu -q -x > gpurun_out/r3c/pytest_win.txt 2>&1; tail -15 gpurun_out/r3c/pytest_win.txt
for v in 0 1 0 1; do
  TBS_WIN=$v timeout 300 python bench.py --no-cpu-baseline --workload sdh_uniform_2m_16k --steps 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('win=$v', round(d['value'],1), d['roofline']['frac'], d['roofline']['kernel_ms_avg'], d['ms_per_step'])"
done
