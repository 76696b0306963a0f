# kNN distance-slot order A/B
mkdir -p gpurun_out/r3r
bash tools/ab_run.sh knn_uniform_1m_k8 5 main kam main kam > gpurun_out/r3r/ab.txt 2>&1
cut -c1-95 gpurun_out/r3r/ab.txt
