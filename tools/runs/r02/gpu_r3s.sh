# hd 64K x 512: raster band re-tune at HEAD (TBS_HD_BAND; default 32)
mkdir -p gpurun_out/r3s
for b in 48 32 48 32 40 56; do
  TBS_HD_BAND=$b timeout 300 python bench.py --workload pairmatrix_hd_64k_d512 --steps 10 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('d512 band $b', round(d['ms_per_step'],3), round(d['value'],1), round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])"
done | tee gpurun_out/r3s/bands.txt
