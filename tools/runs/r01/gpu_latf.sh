# Lattice fast-variant split: parity (lattice tests) + A/B of its residency config.
set -x
timeout 900 python -m pytest tests -q -m gpu -x -k "lattice or exact" 2>&1 | tail -3
bash tools/ab_run.sh sdh_lattice_4m 3 main latf2 latf4
