# windowed C4 configs (TBS_WIN=1): R / KA / TP / CTAs per SM
mkdir -p gpurun_out/r3e
export TBS_WIN=1
bash tools/ab_run.sh sdh_uniform_2m_16k 3 main wb wc wd we wf wg > gpurun_out/r3e/ab.txt 2>&1
cut -c1-100 gpurun_out/r3e/ab.txt
