# SDH 1M config A/B (KA, TP, CTAs/SM, partner-loop unroll) + the NCCL world-1 combine test
set -x
mkdir -p gpurun_out/r2n
timeout 600 python -m pytest tests/test_gpu_fused.py -m gpu -q -k nccl > gpurun_out/r2n/pytest_nccl.txt 2>&1
tail -3 gpurun_out/r2n/pytest_nccl.txt
bash tools/ab_run.sh sdh_uniform_1m 10 main ka16m2 pu2 tp2k ka16m2tp512 ka4m4 main > gpurun_out/r2n/ab_sdh1m.txt 2>&1
cat gpurun_out/r2n/ab_sdh1m.txt
