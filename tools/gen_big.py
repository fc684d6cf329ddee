"""Generate C4 / C5 on the GPU and print shape statistics, time and peak memory."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import graphgen as gg
for cfg in sys.argv[1:]:
    torch.cuda.reset_peak_memory_stats()
    t = time.time()
    g = gg.make(cfg, device="cuda", weights=(cfg != "C5"))
    torch.cuda.synchronize()
    dt = time.time() - t
    deg = g.degrees()
    print(f"{cfg}: n={g.n} m={g.m} gen={dt:.1f}s peak={torch.cuda.max_memory_allocated()/2**30:.1f}GiB "
          f"zero-out={float((deg == 0).float().mean()):.3f} max-out={int(deg.max())} "
          f"top5={[int(x) for x in torch.topk(deg, 5).values]} frac_edges_deg>1024={float(deg[deg>1024].sum())/g.m:.3f}",
          flush=True)
    del g, deg
    torch.cuda.empty_cache()
