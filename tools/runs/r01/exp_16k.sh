for r in 0 1; do
  TBS_LOG2R=$r timeout 300 python bench.py --workload sdh_uniform_2m_16k --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('log2r', $r, d['value'], d['ms_per_step'])"
done
