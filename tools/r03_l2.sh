#!/bin/bash
# The expand's L2 roofline: the chip's random-request ceiling (gather_bench), the
# expand traffic passes with L2 request counts, then the bench lines (which read
# both) for C1-C5.
set -u
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
O=gpurun_out/fin5; mkdir -p $O profiles/r03
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gb tools/gather_bench.cu && /tmp/gb > $O/gather_bench.txt 2>&1
cat $O/gather_bench.txt | tail -22
python tools/l2_ceiling.py $O/gather_bench.txt > profiles/r03/l2_ceiling.json; head -3 profiles/r03/l2_ceiling.json
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex.sum,lts__t_sectors_srcunit_tex.sum
tr() { cfg=$1; algs=$2; tag=${cfg}_${algs//,/+}
  timeout 1800 ncu --metrics $M --cache-control none --clock-control none -k regex:expand_warp --csv \
    --log-file $O/traffic_$tag.csv python tools/prof_run.py --config $cfg --algs $algs --json $O/traffic_$tag.stats.json > $O/traffic_$tag.log 2>&1
  python tools/traffic_summary.py $O/traffic_$tag.csv $O/traffic_$tag.stats.json > profiles/r03/expand_traffic_$tag.json
  python -c "import json; d=json.load(open('profiles/r03/expand_traffic_$tag.json')); print('$tag', {k: round(v,3) for k,v in d.items() if k.startswith('l2') or k.startswith('dram_over')})"
  gzip -f $O/traffic_$tag.csv; }
tr C2 bfs,sssp,cc; tr C3 bfs,sssp; tr C1 bfs,sssp,cc; tr C5 bfs; tr C4 sssp
b() { name=$1; shift; timeout ${T:-900} python bench.py --json-out $O/bench_$name.json "$@" > $O/bench_$name.log 2>&1; \
  python -c "import json; d=json.load(open('$O/bench_$name.json')); r=d['roofline'] or {}; l=r.get('l2') or {}; print('$name', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, 'frac', round(r.get('frac',0),3), 'l2', round(l.get('achieved',0),1), round(l.get('frac',0),3), 'e2e', (d.get('e2e') or {}).get('value'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>/dev/null || { echo "$name FAILED"; tail -5 $O/bench_$name.log; }; }
b c2
b c3 --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline
T=1800 b c4 --config C4 --algs sssp --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
T=1800 b c5 --config C5 --algs bfs --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
b c1 --config C1 --steps 20 --warmup 5 --no-e2e
mkdir -p $O/prof; cp $O/bench_*.json profiles/r03/*.json $O/prof/ 2>/dev/null; du -sh $O
