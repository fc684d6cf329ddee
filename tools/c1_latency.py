"""Where the time of a small-graph call goes (C1 by default): per-call device
time in graph mode and host-loop mode, and with ETG_PROFILE the summed kernel
time (expand + scan) -- the rest is launch / graph overhead."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C1"
dev = torch.device("cuda:0")
g = gg.make(cfg, device=dev)
srcs = gg.sample_sources(g, 8, 4242)
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device=dev)
for name, flags in (("graph", 0), ("hostloop", etg.HOST_LOOP), ("profile", etg.PROFILE)):
    G = etg.Graph(o, c, w, n=g.n, flags=fl | flags, sssp_delta="auto")
    for alg in (etg.BFS, etg.SSSP):
        for s in srcs[:2]:
            G.run(alg, s)                     # warm-up (graph build)
        ms = it = sc = ex = 0.0
        for s in srcs:
            _, st = G.run(alg, s)
            ms += st.ms
            it += st.iterations
            sc += st.scan_ms
            ex += st.expand_ms
        k = len(srcs)
        print(f"{cfg} {name:9s} {'bfs' if alg == 0 else 'sssp'}: {1e3 * ms / k:7.1f} us/call, {it / k:5.1f} iterations, "
              f"{1e3 * ms / max(it, 1):6.1f} us/iteration" +
              (f"; kernels: expand {1e3 * ex / k:.1f} + scan {1e3 * sc / k:.1f} us/call" if flags == etg.PROFILE else ""))
