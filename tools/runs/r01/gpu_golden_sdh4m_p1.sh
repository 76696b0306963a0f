# One pair-balanced half of the 4M SDH golden with the CPU oracle on the GPU box's host cores.
python tools/make_goldens.py --part 1 2 gpurun_out sdh_uniform_n4194304_nb256_seed6
