"""Synchronous model of the SSSP schedules (numpy): relaxations and iterations
of the paper's schedule (Delta = 0), the wave (threshold + Delta per
iteration) and a light/heavy split of the wave (Delta-stepping-like: edges
with w <= Delta relaxed on every activation, heavier ones only once the vertex
is Delta behind the wave; a second snapshot per vertex).  Distances are
checked against scipy's Dijkstra.  Usage: python tools/sssp_schedule_sim.py [C1|LJ-small|T14]"""
import os
import sys

import numpy as np
import scipy.sparse as sp
from scipy.sparse.csgraph import dijkstra

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C1"
g = gg.make(cfg)
off, col, w = (x.astype(np.int64) for x in g.numpy())
n, deg = g.n, np.diff(off)
src_of = np.repeat(np.arange(n), deg)
s = gg.sample_sources(g, 1, 4242)[0]
INF = 1 << 40
ref = dijkstra(sp.csr_matrix((w.astype(np.float64), col, off), shape=(n, n)), indices=s)
ref = np.where(np.isinf(ref), INF, ref).astype(np.int64)
m_reach = deg[ref < INF].sum()


def run(delta, light_heavy):
    lab = np.full(n, INF)
    lab[s] = 0
    snap = np.full(n, INF)
    snap_h = np.full(n, INF)
    th = delta if delta else INF
    it = gathers = reads = 0
    while True:
        ml = lab != snap
        mh = (lab != snap_h) if light_heavy else np.zeros(n, bool)
        la = ml & (lab < th)
        ha = (mh & (lab + delta < th)) if light_heavy else np.zeros(n, bool)
        pend = (ml & ~la) | (mh & ~ha)
        if not (la.any() or ha.any()):
            if not pend.any():
                break
            th = np.where(ml & ~la, lab, lab + delta)[pend].min() + delta
            continue
        it += 1
        snap[la] = lab[la]
        snap_h[ha] = lab[ha]
        e = (la | ha)[src_of]
        rel = (e & ((la[src_of] & (w <= delta)) | (ha[src_of] & (w > delta)))) if light_heavy else e
        reads += e.sum()
        gathers += rel.sum()
        np.minimum.at(lab, col[rel], lab[src_of[rel]] + w[rel])
        if delta:
            th += delta
    assert np.array_equal(lab, ref)
    return it, gathers / m_reach, reads / m_reach


for d in (0, 6, 12, 16, 24):
    print(cfg, "Delta", d, "wave        iterations %d  gathers %.2f  edge reads %.2f (x m_reached)" % run(d, False))
    if d:
        print(cfg, "Delta", d, "light/heavy iterations %d  gathers %.2f  edge reads %.2f (x m_reached)" % run(d, True))
