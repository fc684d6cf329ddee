"""Where the e2e (etg_run_host) time goes on one config: pure H2D of the same
pinned buffers, the resident traversal, and the whole run_host call."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_wangzlg19_b200 as etg  # noqa: E402

dev = torch.device("cuda:0")
flags = int(sys.argv[1]) if len(sys.argv) > 1 else 0
g = gg.make("C2", device="cpu")
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device="cpu")
o, c, w = o.pin_memory(), c.pin_memory(), w.pin_memory()
s = gg.first_source(g)
hout = torch.empty(g.n, dtype=torch.int32).pin_memory()
scratch = torch.empty(etg.host_scratch_bytes(g.n, g.m, True, 32), dtype=torch.uint8, device=dev)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for alg, name, ww in ((etg.BFS, "bfs", None), (etg.SSSP, "sssp", w)):
    for rep in range(4):
        torch.cuda.synchronize()
        ev0.record()
        t0 = time.perf_counter()
        etg.run_host(alg, o, c, ww, s, hout, scratch, flags=flags, sssp_delta=12)
        ev1.record()
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        if rep:
            print(f"{name} run_host flags={flags}: {ev0.elapsed_time(ev1):.2f} ms (host {1e3*(t1-t0):.2f} ms)")
    d_o, d_c = torch.empty_like(o, device=dev), torch.empty_like(c, device=dev)
    d_w = torch.empty_like(w, device=dev) if ww is not None else None
    for rep in range(3):
        torch.cuda.synchronize()
        ev0.record()
        d_o.copy_(o, non_blocking=True)
        d_c.copy_(c, non_blocking=True)
        if d_w is not None:
            d_w.copy_(w, non_blocking=True)
        d_h = torch.empty(g.n, dtype=torch.int32, device=dev)
        hout.copy_(d_h, non_blocking=True)
        ev1.record()
        torch.cuda.synchronize()
        nb = o.numel() * 4 + c.numel() * 4 + (w.numel() * 4 if ww is not None else 0)
        print(f"{name} pure copies {nb/1e9:.3f} GB H2D + 16.8 MB D2H: {ev0.elapsed_time(ev1):.2f} ms "
              f"({nb / ev0.elapsed_time(ev1) / 1e6:.1f} GB/s)")
