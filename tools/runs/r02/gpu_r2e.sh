# C1 small-kernel probe: replication R, occupancy, config threshold; CTA trace; ncu of one launch
set -x
mkdir -p gpurun_out/r2e
for r in 5 4 3 2 1 0; do TBS_LOG2R=$r python tools/c1_probe.py >> gpurun_out/r2e/c1_probe.jsonl 2>&1; done
for o in 1 2 3; do TBS_OCC=$o python tools/c1_probe.py >> gpurun_out/r2e/c1_probe.jsonl 2>&1; done
TBS_SMALL_ITEMS=0 python tools/c1_probe.py >> gpurun_out/r2e/c1_probe.jsonl 2>&1
TBS_TRACE=1 python tools/c1_probe.py > gpurun_out/r2e/c1_trace.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 20 -c 1 -o gpurun_out/r2e/prof_c1 python tools/c1_probe.py > gpurun_out/r2e/ncu_c1.log 2>&1
