set -x
timeout 900 python -m pytest tests -q -m gpu -x -k "lattice or exact or sqrt" 2>&1 | tail -3
./build/sqrt_bound
bash tools/ab_run.sh sdh_lattice_4m 3 main
bash tools/ab_run.sh sdh_uniform_1m 5 main
