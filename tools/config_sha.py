"""Record the SHA-256 of every config's generated CSR (off, col and w as the
oracle reads them: uint64 / uint32 / uint32; graphgen.Graph.sha256) --
input provenance.  Small configs on the CPU; with --device cuda
the big ones on the GPU.  Usage: python tools/config_sha.py [--device cuda]
[--configs C1,T12,...] [--out tests/golden/config_sha256.json]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--device", default="cpu")
ap.add_argument("--configs", default="T12,T14,C1,LJ-small")
ap.add_argument("--out", default=None)
a = ap.parse_args()
res = {}
for cfg in a.configs.split(","):
    for sym in (False, True):
        g = gg.make(cfg, device=a.device, weights=not sym, symmetric=sym)
        res[g.name + ("" if sym else "+w")] = {"n": g.n, "m": g.m, "sha256": g.sha256()}
        print(cfg, "sym" if sym else "w", g.n, g.m, res[g.name + ("" if sym else "+w")]["sha256"], flush=True)
        del g
if a.out:
    old = {}
    if os.path.exists(a.out):
        old = json.load(open(a.out))
    old.update(res)
    with open(a.out, "w") as f:
        json.dump(old, f, indent=1, sort_keys=True)
