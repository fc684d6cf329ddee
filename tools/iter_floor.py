"""Per-iteration floor of the traversal loop: BFS on a directed path of L
vertices runs L iterations of one active vertex each, so time / L is the
fixed cost of one Proc. 1 iteration (expand + scan + loop control), graph mode
and host loop."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402

for L in (256, 2048):
    for n_extra in (0, 4_000_000):        # a path inside a graph of n vertices (scan covers all n)
        n = L + n_extra
        off = torch.zeros(n + 1, dtype=torch.int64)
        off[1:L] = torch.arange(1, L)
        off[L:] = L - 1
        col = torch.arange(1, L, dtype=torch.int64)
        o, c, _, fl = etg.csr_to_device(off, col, None, device="cuda")
        for name, flags in (("graph", 0), ("hostloop", etg.HOST_LOOP)):
            G = etg.Graph(o, c, None, n=n, flags=fl | flags)
            G.bfs(0)
            ms = 0.0
            for _ in range(3):
                _, st = G.bfs(0)
                ms += st.ms
            print(f"path L={L} n={n}: {name:8s} {1e3 * ms / 3 / st.iterations:6.2f} us/iteration "
                  f"({st.iterations} iterations)", flush=True)
