# refresh at HEAD: ncu of C4 and the 2PCF pair kernel, the paper-experiment ablations, the partition proxy
set -x
O=gpurun_out/r3h
mkdir -p $O
for wl in sdh_uniform_2m_16k pcf_clustered_4m; do
  ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o /tmp/prof_$wl \
    python bench.py --workload $wl --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_$wl.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$wl.ncu-rep > $O/ncu_summary_$wl.txt 2>&1
  ncu -i /tmp/prof_$wl.ncu-rep --page details > $O/ncu_details_$wl.txt 2>&1
done
timeout 900 python tools/ablations.py > $O/ablations.jsonl 2>&1
timeout 900 python tools/partition_balance.py > $O/partition_balance.jsonl 2>&1
ls -la $O
