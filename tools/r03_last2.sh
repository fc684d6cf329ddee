#!/bin/bash
# Round end, final code: smoke, the GPU suite, bench lines C2 (default) and C3.
O=gpurun_out/last2; mkdir -p $O/prof
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 2000 python -m pytest tests -m gpu -q -x > $O/gputest.log 2>&1; tail -2 $O/gputest.log
python bench.py --json-out $O/prof/bench_c2.json > $O/bench_c2.log 2>&1
python bench.py --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline --json-out $O/prof/bench_c3.json > $O/bench_c3.log 2>&1
for c in c2 c3; do python -c "import json; d=json.load(open('$O/prof/bench_$c.json')); r=d['roofline']; print('$c', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, round(r['frac'],3), round((r.get('l2') or {}).get('frac',0),3), (d.get('e2e') or {}).get('value'), d['clocks'])"; done
