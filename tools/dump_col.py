import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np, graphgen as gg
g = gg.make("C2", device="cuda", weights=False)
c = g.col[: 64 << 20].to(torch.int32).cpu().numpy()
c.tofile(sys.argv[1])
# also a shuffled copy (same multiset of targets, no locality)
rng = np.random.default_rng(1)
rng.shuffle(c)
c.tofile(sys.argv[2])
print("m", g.m)
