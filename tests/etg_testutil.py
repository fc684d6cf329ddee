"""Helpers shared by the test modules (no method arithmetic)."""
import json
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def to_etg(g, K=32, flags=0, symmetric=None, device="cuda", force_u64=False, sssp_delta=0):
    """graphgen.Graph -> paper_conf_ipps_wangzlg19_b200.Graph on the device."""
    import torch
    import paper_conf_ipps_wangzlg19_b200 as etg
    o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device=device)
    if force_u64:
        o = g.off.to(device=device, dtype=torch.int64).contiguous()
    sym = g.symmetric if symmetric is None else symmetric
    return etg.Graph(o, c, w, n=g.n, K=K, flags=flags | fl, symmetric=sym, validate=True,
                     sssp_delta=sssp_delta)


def sssp_certificate_gpu(g, s, dist, chunk=1 << 27):
    """Shortest-path certificate on the device (a property that characterises
    the saturated distances uniquely for weights >= 1):
    dist[s] = 0; for every edge (u,v) with dist[u] finite, dist[v] <= sat(dist[u]+w);
    every reached v != s has a tight in-edge.  Returns None or a message."""
    import torch
    INF, CAP = 0xFFFFFFFF, 0xFFFFFFFE
    d = dist.to(torch.int64) & 0xFFFFFFFF
    if int(d[s]) != 0:
        return "dist[s] != 0"
    deg = g.off[1:] - g.off[:-1]
    tight = torch.zeros(g.n, dtype=torch.bool, device=d.device)
    starts = torch.arange(g.n, device=d.device)
    for lo in range(0, g.m, chunk):
        hi = min(g.m, lo + chunk)
        # sources of edges lo..hi
        src = torch.searchsorted(g.off, torch.arange(lo, hi, device=d.device), right=True) - 1
        dst = g.col[lo:hi].to(torch.int64)
        w = g.w[lo:hi].to(torch.int64)
        du = d[src]
        fin = du != INF
        cand = torch.clamp(du + w, max=CAP)
        dv = d[dst]
        if bool((fin & (dv > cand)).any()):
            return f"edge relaxable in [{lo},{hi})"
        tight[dst[fin & (dv == cand)]] = True
        del src, dst, w, du, fin, cand, dv
    reached = d != INF
    reached[s] = False
    if bool((reached & ~tight).any()):
        return "reached vertex without a tight in-edge"
    return None
