# Round-end verification at HEAD: GPU parity suite, smoke, bench (own arm + reference arm).
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu -x -rA 2>&1 | grep -E "passed|failed|error|golden part" | tail -8 | tee gpurun_out/final_pytest.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py --steps 5 --warmup 3 2>&1 | tail -1 | tee gpurun_out/final_bench.json | cut -c1-600
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 2>&1 | tail -1 | cut -c1-400
