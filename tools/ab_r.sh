# A/B of the replication factor R = 2^TBS_LOG2R and the small-problem threshold
for nb in 768 1024 2048 4096 8192 16384; do
  for r in 5 4 3 2 1 0; do
    TBS_LOG2R=$r python - <<PY
import math, numpy as np, torch, sys
sys.path.insert(0, '.')
import paper_conf_icpp_pitaksirianannt16_b200 as tbs, tbs_inputs as g
p = torch.from_numpy(g.uniform(1 << 20, 2)).cuda()
w = float(np.float32(math.sqrt(3) / $nb))
try:
    for _ in range(2): tbs.sdh(p, w, $nb)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); tbs.sdh(p, w, $nb); b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b); print("nb", $nb, "log2r", $r, "ms", round(ms, 2), "Gpairs/s", round(p.shape[0]*(p.shape[0]-1)/2/ms/1e6, 1))
except Exception as e:
    print("nb", $nb, "log2r", $r, "skip", str(e)[:60])
PY
  done
done
for thr in 2 8 16 32; do
  TBS_SMALL_ITEMS=$thr python - <<PY
import math, numpy as np, torch, sys
sys.path.insert(0, '.')
import paper_conf_icpp_pitaksirianannt16_b200 as tbs, tbs_inputs as g
for m in (16384, 32768, 65536, 131072, 262144):
    p = torch.from_numpy(g.uniform(m, 1)).cuda(); w = float(np.float32(math.sqrt(3) / 64))
    for _ in range(3): tbs.sdh(p, w, 64)
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); tbs.sdh(p, w, 64); b.record(); torch.cuda.synchronize(); best = min(best, a.elapsed_time(b))
    print("small_thr", $thr, "n", m, "ms", round(best, 3), "Gpairs/s", round(m*(m-1)/2/best/1e6, 1))
PY
done
