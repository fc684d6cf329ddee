#!/bin/bash
# Last evidence pass of the round (final kernels): expand traffic with L2 request
# counts (C1-C5), bench lines C1-C5 (+ UDC off, N = 2 both partitions, reference
# arm), warm launch list.  Results -> gpurun_out/fin6/prof.
set -u
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
O=gpurun_out/fin6; mkdir -p $O/prof profiles/r03
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex.sum,lts__t_sectors_srcunit_tex.sum
tr() { cfg=$1; algs=$2; tag=${cfg}_${algs//,/+}
  timeout 1800 ncu --metrics $M --cache-control none --clock-control none -k regex:expand_warp --csv \
    --log-file $O/traffic_$tag.csv python tools/prof_run.py --config $cfg --algs $algs --json $O/traffic_$tag.stats.json > $O/traffic_$tag.log 2>&1
  python tools/traffic_summary.py $O/traffic_$tag.csv $O/traffic_$tag.stats.json > profiles/r03/expand_traffic_$tag.json
  cp profiles/r03/expand_traffic_$tag.json $O/prof/
  python tools/launch_top.py $O/traffic_$tag.csv > $O/prof/top_$tag.txt
  python -c "import json; d=json.load(open('profiles/r03/expand_traffic_$tag.json')); print('$tag', {k: round(v,3) for k,v in d.items() if isinstance(v,float) and (k.startswith('l2') or k.startswith('dram'))})"
  gzip -f $O/traffic_$tag.csv; }
tr C2 bfs,sssp,cc; tr C3 bfs,sssp; tr C1 bfs,sssp,cc; tr C5 bfs; tr C4 sssp
b() { name=$1; shift; timeout ${T:-900} python bench.py --json-out $O/bench_$name.json "$@" > $O/bench_$name.log 2>&1; cp $O/bench_$name.json $O/prof/ 2>/dev/null; \
  python -c "import json; d=json.load(open('$O/bench_$name.json')); r=d.get('roofline') or {}; l=r.get('l2') or {}; print('$name', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, 'frac', round(r.get('frac',0) or 0,3), 'l2', round(l.get('frac',0) or 0,3), 'e2e', (d.get('e2e') or {}).get('value'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>/dev/null || { echo "$name FAILED"; tail -5 $O/bench_$name.log; }; }
b c2
python bench.py --impl reference --steps 6 --warmup 1 > $O/prof/bench_c2_reference.json 2> $O/bench_c2_reference.err; tail -c 200 $O/prof/bench_c2_reference.json; echo
b c3 --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline
b c3_noudc --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --flags 2
T=1800 b c4 --config C4 --algs sssp --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
T=1800 b c5 --config C5 --algs bfs --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
b c1 --config C1 --steps 20 --warmup 5 --no-e2e
b c2_n2 --gpus 2 --steps 5 --warmup 3
b c2_n2_push --gpus 2 --steps 5 --warmup 3 --push --no-e2e
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan|init_kernel|publish" --csv \
    --log-file $O/launches_warm.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
python tools/launches.py $O/launches_warm.csv 80 > $O/prof/launches_warm.txt 2>&1; head -8 $O/prof/launches_warm.txt
cp $O/launches_warm.csv $O/prof/launches_warm_r03.csv
du -sh $O
