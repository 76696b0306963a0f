# evidence at HEAD after the per-Op slot order: GPU suite, smoke, bench lines, ncu of the SDH pair kernel, launch list
set -x
O=gpurun_out/r3a
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 3000 python -m pytest tests -m gpu -q > $O/pytest_gpu.txt 2>&1
tail -3 $O/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
python bench.py > $O/bench_default.json 2> $O/bench_default.err
B="timeout 900 python bench.py --no-cpu-baseline"
for wl in sdh_uniform_4m sdh_clustered_1m sdh_lattice_4m sdh_uniform_4k pcf_clustered_4m kde_uniform_1m sdh_uniform_2m_16k; do
  S=10; case $wl in sdh_uniform_4m|sdh_lattice_4m|pcf_clustered_4m|sdh_uniform_2m_16k) S=3;; sdh_uniform_4k) S=50;; esac
  $B --workload $wl --steps $S > $O/bench_$wl.json 2> $O/bench_$wl.err
done
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_sdh_uniform_1m.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/launches.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:pair_kernel -s 3 -c 1 -o /tmp/prof_sdh1m \
  python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_sdh1m.log 2>&1
python tools/ncu_summary.py /tmp/prof_sdh1m.ncu-rep > $O/ncu_summary_sdh_uniform_1m.txt 2>&1
ncu -i /tmp/prof_sdh1m.ncu-rep --page details > $O/ncu_details_sdh_uniform_1m.txt 2>&1
ls -la $O
