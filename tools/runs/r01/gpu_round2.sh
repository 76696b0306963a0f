set -x
timeout 1200 python -m pytest tests -q -m gpu -x 2>&1 | tail -3
bash tools/sanitize.sh
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 3 --warmup 3 2>&1 | tail -2 | cut -c1-300
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 2>&1 | tail -1 | cut -c1-400
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
