"""Per-iteration fixed cost of the partitioned loop (etg_comm handles): BFS on a
directed path of L vertices (one active vertex per iteration), P ranks as
threads of this process on one GPU; compared with the single-GPU graph loop.
Prints us per iteration (the library's per-call device time, max over ranks)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402
from paper_conf_ipps_wangzlg19_b200 import dist as edist  # noqa: E402

L = 1024
n = L
off = torch.zeros(n + 1, dtype=torch.int64)
off[1:L] = torch.arange(1, L)
off[L:] = L - 1
col = torch.arange(1, L, dtype=torch.int64)
o, c, _, fl = etg.csr_to_device(off, col, None, device="cuda")
G = etg.Graph(o, c, None, n=n, flags=fl)
G.bfs(0)
_, st = G.bfs(0)
print(f"single GPU, CUDA-graph loop: {1e3 * st.ms / st.iterations:7.2f} us/iteration")
Gh = etg.Graph(o, c, None, n=n, flags=fl | etg.HOST_LOOP)
Gh.bfs(0)
_, st = Gh.bfs(0)
print(f"single GPU, host-driven loop: {1e3 * st.ms / st.iterations:7.2f} us/iteration")
for P in (1, 2, 4):
    for exchange in ("dest",):
        parts = edist.local_partitions(off, col, None, n, P, exchange=exchange)
        edist.run_local(parts, etg.BFS, 0)
        _, st = edist.run_local(parts, etg.BFS, 0)
        print(f"P = {P} ranks (threads), {exchange}: {1e3 * st.ms / st.iterations:7.2f} us/iteration "
              f"({st.iterations} loop trips)", flush=True)
        for p in parts:
            p.close()
