#!/bin/bash
# Round end check: smoke, the whole GPU suite, the default bench line; the
# UDC-off C3 line with its own expand traffic capture.
mkdir -p gpurun_out/last/prof
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" > gpurun_out/last/smoke.log 2>&1; tail -2 gpurun_out/last/smoke.log
timeout 2000 python -m pytest tests -m gpu -q -x --durations=5 > gpurun_out/last/gputest.log 2>&1; tail -12 gpurun_out/last/gputest.log
python bench.py > gpurun_out/last/bench_default.json 2> gpurun_out/last/bench_default.err; python -c "import json; d=json.load(open('gpurun_out/last/bench_default.json')); print('default', d['value'], d['roofline']['frac'], (d['roofline'].get('l2') or {}).get('frac'), d['e2e']['value'], d['clocks'])"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex.sum,lts__t_sectors_srcunit_tex.sum
O=gpurun_out/last
timeout 1500 ncu --metrics $M --cache-control none --clock-control none -k regex:expand_warp --csv --log-file $O/traffic_noudc.csv \
   python tools/prof_run.py --config C3 --algs bfs,sssp --flags 34 --json $O/traffic_noudc.stats.json > $O/traffic_noudc.log 2>&1
python tools/traffic_summary.py $O/traffic_noudc.csv $O/traffic_noudc.stats.json > profiles/r03/expand_traffic_C3_bfs+sssp_flags2.json
cp profiles/r03/expand_traffic_C3_bfs+sssp_flags2.json $O/prof/
python bench.py --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --flags 2 --json-out $O/prof/bench_c3_noudc.json > $O/noudc.log 2>&1
python -c "import json; d=json.load(open('$O/prof/bench_c3_noudc.json')); r=d['roofline']; print('noudc', d['value'], r['frac'], r.get('traffic'), (r.get('l2') or {}).get('frac'))"
