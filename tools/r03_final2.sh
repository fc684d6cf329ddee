#!/bin/bash
# Refresh of the round's evidence after the last scan/expand changes: C2 expand
# traffic, bench lines C1-C5 (+ UDC off, N = 2, reference arm), warm launch
# list, ncu of a dense (vertex-list) and a sparse SSSP scan.
set -u
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
O=gpurun_out/fin4; mkdir -p $O profiles/r03
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
tr() { cfg=$1; algs=$2; tag=${cfg}_${algs//,/+}
  timeout 1500 ncu --metrics $M --cache-control none --clock-control none -k regex:expand_warp --csv \
    --log-file $O/traffic_$tag.csv python tools/prof_run.py --config $cfg --algs $algs --json $O/traffic_$tag.stats.json > $O/traffic_$tag.log 2>&1
  python tools/traffic_summary.py $O/traffic_$tag.csv $O/traffic_$tag.stats.json > profiles/r03/expand_traffic_$tag.json
  python tools/launch_top.py $O/traffic_$tag.csv > $O/top_$tag.txt; head -3 $O/top_$tag.txt
  gzip -f $O/traffic_$tag.csv; }
tr C2 bfs,sssp,cc; tr C3 bfs,sssp
b() { name=$1; shift; timeout ${T:-900} python bench.py --json-out $O/bench_$name.json "$@" > $O/bench_$name.log 2>&1; \
  python -c "import json; d=json.load(open('$O/bench_$name.json')); r=d['roofline'] or {}; print('$name', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, 'frac', round(r.get('frac',0),3), 'traffic', r.get('traffic'), 'e2e', (d.get('e2e') or {}).get('value'), d['clocks'])" 2>/dev/null || { echo "$name FAILED"; tail -5 $O/bench_$name.log; }; }
b c2
python bench.py --impl reference --steps 6 --warmup 1 > $O/bench_c2_reference.json 2> $O/bench_c2_reference.err; tail -c 300 $O/bench_c2_reference.json; echo
b c3 --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline
b c3_noudc --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --flags 2
T=1800 b c4 --config C4 --algs sssp --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
T=1800 b c5 --config C5 --algs bfs --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
b c1 --config C1 --steps 20 --warmup 5 --no-e2e
b c2_n2 --gpus 2 --steps 5 --warmup 3
b c2_n2_push --gpus 2 --steps 5 --warmup 3 --push --no-e2e
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan|init_kernel|publish" --csv \
    --log-file $O/launches_warm.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
python tools/launches.py $O/launches_warm.csv 80 > $O/launches_warm.txt 2>&1; head -8 $O/launches_warm.txt
full() { tag=$1; cfg=$2; algs=$3; k=$4; idx=$5
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s $idx -c 1 -o $O/full_$tag \
     python tools/prof_run.py --config $cfg --algs $algs > $O/full_$tag.log 2>&1
  python tools/ncu_lines.py $O/full_$tag.ncu-rep 25 > $O/full_$tag.lines.txt 2>&1
  ncu -i $O/full_$tag.ncu-rep --page raw --csv > $O/full_$tag.raw.csv 2>/dev/null; gzip -f $O/full_$tag.raw.csv
  python tools/ncu_summary.py $O/full_$tag.raw.csv.gz > $O/full_$tag.summary.json; head -4 $O/full_$tag.summary.json; }
full c2_sssp_scan_dense C2 sssp udc_scan 6
full c2_sssp_scan_sparse C2 sssp udc_scan 16
full c2_sssp_expand_mid C2 sssp expand_warp 3
mkdir -p $O/prof
cp $O/bench_*.json $O/*.lines.txt $O/*.summary.json $O/launches_warm.txt $O/top_*.txt profiles/r03/expand_traffic_C2_bfs+sssp+cc.json profiles/r03/expand_traffic_C3_bfs+sssp.json $O/prof/ 2>/dev/null
rm -f $O/*.ncu-rep
du -sh $O
