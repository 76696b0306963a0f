# slot order A/B: blocked 2x2 (mq4) and diagonal (mq5) for every Op vs the per-Op main
mkdir -p gpurun_out/r3b
for wl in sdh_uniform_1m kde_uniform_1m; do bash tools/ab_run.sh $wl 10 main mq4 mq5 main mq4 mq5; done > gpurun_out/r3b/ab.txt 2>&1
for wl in sdh_lattice_4m pcf_clustered_4m; do bash tools/ab_run.sh $wl 3 main mq4 mq5; done >> gpurun_out/r3b/ab.txt 2>&1
cut -c1-95 gpurun_out/r3b/ab.txt
