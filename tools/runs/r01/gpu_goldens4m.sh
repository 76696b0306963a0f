# Full-size 4M goldens with the CPU oracle on the GPU box's host cores (no GPU use).
set -x
nproc
python tools/make_goldens.py pcf_clustered_n4194304_r0.03_seed3
cp tests/golden/pcf_clustered_n4194304_r0.03_seed3.json gpurun_out/
python tools/make_goldens.py sdh_uniform_n4194304_nb256_seed6
cp tests/golden/sdh_uniform_n4194304_nb256_seed6.json gpurun_out/
