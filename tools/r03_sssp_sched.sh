#!/bin/bash
# SSSP schedule study on C2: wave vs classic near-far, per-iteration trace
mkdir -p gpurun_out
cat > /tmp/sd.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import torch, graphgen as gg, paper_conf_ipps_wangzlg19_b200 as etg
cfg = sys.argv[1]
g = gg.make(cfg, device="cuda")
srcs = gg.sample_sources(g, 4, 4242)
o, c, w, fl = etg.csr_to_device(g.off, g.col, g.w, device="cuda")
for dl in [int(x) for x in sys.argv[2].split(",")]:
    G = etg.Graph(o, c, w, n=g.n, flags=fl, sssp_delta=dl)
    G.sssp(srcs[0])
    ms = it = ed = 0
    for s in srcs:
        _, st = G.sssp(s); ms += st.ms; it += st.iterations; ed += st.edges_processed
    k = len(srcs)
    print(f"{cfg} tune={os.environ.get('ETG_TUNE','0')} delta={dl:4d} iters={it/k:6.1f} edges={ed/k/1e6:8.1f}M ms={ms/k:.3f}", flush=True)
    del G
PY
python /tmp/sd.py C2 0,6,12,24 2>&1 | tee gpurun_out/sched.txt
ETG_TUNE=8192 python /tmp/sd.py C2 4,8,16,32,64,128 2>&1 | tee -a gpurun_out/sched.txt
python tools/iter_trace.py --config C2 --algs sssp --delta 12 > gpurun_out/trace_wave12.txt 2>&1; head -40 gpurun_out/trace_wave12.txt
ETG_TUNE=8192 python tools/iter_trace.py --config C2 --algs sssp --delta 32 > gpurun_out/trace_nf32.txt 2>&1; head -80 gpurun_out/trace_nf32.txt
python tools/iter_trace.py --config C2 --algs cc,bfs > gpurun_out/trace_cc_bfs.txt 2>&1; cat gpurun_out/trace_cc_bfs.txt
