import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import graphgen as gg, oracle, paper_conf_ipps_wangzlg19_b200 as etg
gs = gg.make("T12", device="cuda", symmetric=True, weights=False)
soff, scol, _ = gs.to("cpu").numpy()
for K in (32, 4):
    o2, c2, _, fl2 = etg.csr_to_device(gs.off, gs.col, None)
    Gs = etg.Graph(o2, c2, None, n=gs.n, K=K, flags=fl2, symmetric=True)
    ok = np.array_equal(etg.to_u32_numpy(Gs.cc()[0]), oracle.cc(soff, scol))
    print("K", K, "cc ok", ok, flush=True)
