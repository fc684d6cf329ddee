"""Helpers shared by the test modules (no method arithmetic)."""
import json
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def to_etg(g, K=32, flags=0, symmetric=None, device="cuda", force_u64=False):
    """graphgen.Graph -> paper_conf_ipps_wangzlg19_b200.Graph on the device."""
    import torch
    import paper_conf_ipps_wangzlg19_b200 as etg
    o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device=device)
    if force_u64:
        o = g.off.to(device=device, dtype=torch.int64).contiguous()
    sym = g.symmetric if symmetric is None else symmetric
    return etg.Graph(o, c, w, n=g.n, K=K, flags=flags | fl, symmetric=sym, validate=True)
