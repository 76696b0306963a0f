# kNN (k = 8) config A/B: anchors per thread x resident CTAs
mkdir -p gpurun_out/r3q
bash tools/ab_run.sh knn_uniform_1m_k8 5 main k4m3 k2m3 k2m4 main > gpurun_out/r3q/ab.txt 2>&1
cut -c1-95 gpurun_out/r3q/ab.txt
