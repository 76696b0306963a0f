import math, numpy as np, torch, sys
sys.path.insert(0, '.')
import paper_conf_icpp_pitaksirianannt16_b200 as tbs, tbs_inputs as g
p = torch.from_numpy(g.uniform(4096, 1)).cuda()
w = float(np.float32(math.sqrt(3) / 64))
for _ in range(3): tbs.sdh(p, w, 64)
torch.cuda.synchronize()
