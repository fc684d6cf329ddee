#!/bin/bash
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
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "far:ETG_X=0"
python /tmp/sd.py C2 0,6,8,12,16 2>&1
ETG_TUNE=8192 python /tmp/sd.py C2 8,16,32 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan" --csv --log-file gpurun_out/launches_far.csv python tools/prof_run.py --algs sssp > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_far.csv 60 2>&1 | head -50
