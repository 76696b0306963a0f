set -x
mkdir -p gpurun_out/r2l
TBS_HOST_TRACE=1 timeout 300 python tools/c1_e2e.py > gpurun_out/r2l/c1_e2e_plans.json 2> gpurun_out/r2l/c1_e2e_plans.err
TBS_NO_PLANS=1 timeout 300 python tools/c1_e2e.py > gpurun_out/r2l/c1_e2e_noplans.json 2>&1
