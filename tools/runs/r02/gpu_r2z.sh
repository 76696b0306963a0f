# anchor-major slot order (mq1) vs main on the other pair-engine workloads
mkdir -p gpurun_out/r2z
for wl in pcf_clustered_4m sdh_lattice_4m sdh_uniform_2m_16k; do bash tools/ab_run.sh $wl 3 main mq1 main mq1; done > gpurun_out/r2z/ab.txt 2>&1
for wl in kde_uniform_1m sdh_clustered_1m sdh_uniform_4k; do bash tools/ab_run.sh $wl 10 main mq1 main mq1; done >> gpurun_out/r2z/ab.txt 2>&1
cut -c1-95 gpurun_out/r2z/ab.txt
