#!/bin/bash
# Final code: smoke, the GPU suite, one default bench line.
O=gpurun_out/last3; mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 2000 python -m pytest tests -m gpu -q -x > $O/gputest.log 2>&1; tail -2 $O/gputest.log
python bench.py --json-out $O/bench_c2.json > $O/bench_c2.log 2>&1
python -c "import json; d=json.load(open('$O/bench_c2.json')); r=d['roofline']; print('c2', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, round(r['frac'],3), round((r.get('l2') or {}).get('frac',0),3), d['clocks'])"
