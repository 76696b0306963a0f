# Round-2 final evidence run at HEAD: full GPU suite + smoke, every bench line (clock records),
# the default line with its CPU baseline and the reference arm, ncu of the dominant kernels,
# the launch list, sanitizers, peaks and the Fig. 7 / Fig. 9 ablations.
set -x
O=gpurun_out/final
mkdir -p $O/san
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 3600 python -m pytest tests -m gpu -q > $O/pytest_gpu.txt 2>&1
tail -3 $O/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err
B="timeout 900 python bench.py --no-cpu-baseline"
for wl in sdh_uniform_4m sdh_clustered_1m sdh_uniform_2m_16k sdh_lattice_4m sdh_uniform_4k pcf_clustered_4m pairmatrix_64k kde_uniform_1m knn_uniform_1m_k8 pairmatrix_hd_64k_d64 pairmatrix_hd_64k_d512; do
  S=10; case $wl in sdh_uniform_4m|sdh_lattice_4m|pcf_clustered_4m|sdh_uniform_2m_16k) S=3;; sdh_uniform_4k) S=3000;; esac
  $B --workload $wl --steps $S > $O/bench_$wl.json 2> $O/bench_$wl.err
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_sdh_uniform_1m.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/launches.log 2>&1
# ncu reports stay on the box (gpurun copies back <= 64 MiB): keep their summaries and details
for wl in sdh_uniform_1m sdh_uniform_2m_16k pcf_clustered_4m; do
  ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o /tmp/prof_$wl \
    python bench.py --workload $wl --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_$wl.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$wl.ncu-rep > $O/ncu_summary_$wl.txt 2>&1
  ncu -i /tmp/prof_$wl.ncu-rep --page details > $O/ncu_details_$wl.txt 2>&1
done
ncu --set full --clock-control none --import-source on -k regex:"pair_kernel" -s 20 -c 1 -o /tmp/prof_c1 python tools/c1_probe.py > $O/ncu_c1.log 2>&1
python tools/ncu_summary.py /tmp/prof_c1.ncu-rep > $O/ncu_summary_c1.txt 2>&1
du -sh $O
./tools/peaks > $O/peaks.json 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ablate_intra tools/ablate_intra.cu && /tmp/ablate_intra > $O/ablate_intra.jsonl 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/sanitize_driver.py 2500 > $O/san/sanitize_$tool.log 2>&1
  echo "$tool exit $?"
done
timeout 300 python tools/c1_e2e.py > $O/c1_e2e.json 2>&1
timeout 900 python tools/partition_balance.py > $O/partition_balance.jsonl 2>&1
timeout 900 python tools/ablations.py > $O/ablations.jsonl 2>&1
ls -la $O
