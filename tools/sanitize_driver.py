"""Small calls of every entry point, for compute-sanitizer (memcheck/racecheck/synccheck/initcheck)."""
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_pitaksirianannt16_b200 as tbs  # noqa: E402
import tbs_inputs as g  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 2500
p = torch.from_numpy(g.clustered(n, 1)).cuda()
lat = torch.from_numpy(g.lattice(13, 2)[:n]).cuda()
w = float(np.float32(math.sqrt(3) / 64))
out = []
for mode in (None, "lane", "cta", "global"):
    out.append(tbs.sdh(p, w, 64, hist_mode=mode).sum().item())
    out.append(tbs.sdh(lat, 0.5, 64, lattice=True, hist_mode=mode).sum().item())
out.append(tbs.sdh(p, w, 5000).sum().item())                 # R = 4 / 2 replicas
out.append(tbs.sdh(p, w, 64, rows=(100, 1900)).sum().item())  # row range, masked items
out.append(tbs.sdh(p, w, 64, force_clamp=True).sum().item())
out.append(tbs.pcf(p, 0.05).item())
out.append(tbs.pcf(p, 0.05, rows=(7, 2000)).item())
out.append(float(tbs.pairmatrix(p[:1001], 1.0).sum().item()))
out.append(float(tbs.pairmatrix(p[:1000], 1.0, kernel="dist").sum().item()))
out.append(tbs.sdh(lat, 0.75, 80, lattice=True).sum().item())     # fast lattice variant, m = 3
out.append(tbs.sdh(lat, 0.75, 7, lattice=True).sum().item())      # clamped two-sided fp32 variant
out.append(tbs.sdh(lat, 0.09375, 256, lattice=True).sum().item())  # one-sided fp32 variant (X = 669)
sink, csink = tbs.PeerSink(64), tbs.PeerSink(1)                    # fused combine (world 1)
out.append(tbs.sdh(p, w, 64, sink=sink).sum().item())
out.append(tbs.sdh(lat, 0.5, 64, lattice=True, hist_mode="global", sink=sink).sum().item())
out.append(tbs.pcf(p, 0.05, rows=(7, 2000), sink=csink).item())
sink.close()
csink.close()
out.append(float(tbs.kde(p, 1.0).item()))
out.append(float(tbs.knn(p, 8)[1].sum().item()))
out.append(float(tbs.knn(p, 5, rows=(3, 1800))[1].sum().item()))
xb = torch.from_numpy(g.uniform(777, 4, 96)).cuda().to(torch.bfloat16)   # hd: CTA pairs, ragged n
out.append(float(tbs.pairmatrix_hd(xb, 0.01).sum().item()))
out.append(float(tbs.pairmatrix_hd(xb, 0.01, rows=(130, 419)).sum().item()))
out.append(float(tbs.pairmatrix_hd(xb[:700], 0.01, kernel="dist").sum().item()))
out.append(float(tbs.rdf(p, w, 64, 1.0).sum().item()))                 # RDF (NEXT-1)
out.append(float(tbs.rdf(lat, 0.5, 64, 2197.0, lattice=True, rows=(5, 1500)).sum().item()))
out.append(tbs.sdh(lat, 0.5, 64, lattice=True, validate=True).sum().item())   # TBS_VALIDATE
big = torch.from_numpy(g.uniform(40000, 3)).cuda()                # main (non-small) tile config
out.append(tbs.sdh(big, w, 64).sum().item())
torch.cuda.synchronize()
print("sanitize driver ok", len(out), out[:3])
