# host-buffer small path: per-phase host time (TBS_HOST_TRACE)
mkdir -p gpurun_out/r3j
TBS_HOST_TRACE=1 timeout 300 python tools/c1_e2e.py > gpurun_out/r3j/c1_e2e.json 2> gpurun_out/r3j/c1_e2e.err
cat gpurun_out/r3j/c1_e2e.json; cat gpurun_out/r3j/c1_e2e.err
