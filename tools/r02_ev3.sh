set -u
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
O=gpurun_out/ev3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q 2>&1 | tail -3
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 1200 ncu --metrics $M --cache-control none --clock-control none -k regex:expand_warp --csv \
    --log-file $O/traffic_C4_sssp.csv python tools/prof_run.py --config C4 --algs sssp --json $O/traffic_C4_sssp.stats.json > $O/traffic_C4_sssp.log 2>&1
python tools/traffic_summary.py $O/traffic_C4_sssp.csv $O/traffic_C4_sssp.stats.json > $O/expand_traffic_C4_sssp.json; gzip -f $O/traffic_C4_sssp.csv
cat $O/expand_traffic_C4_sssp.json | head -12
mkdir -p profiles/r02 && cp $O/expand_traffic_C4_sssp.json profiles/r02/
b() { name=$1; shift; timeout ${T:-900} python bench.py --json-out $O/bench_$name.json "$@" > $O/bench_$name.log 2>&1; \
  python -c "import json; d=json.load(open('$O/bench_$name.json')); r=d['roofline'] or {}; print('$name', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, 'frac', round(r.get('frac',0),3), 'traffic', r.get('traffic'), 'e2e', (d.get('e2e') or {}).get('value'))" 2>/dev/null || { echo "$name FAILED"; tail -5 $O/bench_$name.log; }; }
T=1500 b c4 --config C4 --algs sssp --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
b c2 --no-cpu-baseline
for t in 0 1024; do ETG_TUNE=$t python tools/c1_latency.py C1 > $O/c1_tune$t.txt 2>&1; cat $O/c1_tune$t.txt; done
ETG_TUNE=1024 python tools/c1_latency.py T14 2>&1 | grep -v profile
python tools/c1_latency.py T14 2>&1 | grep -v profile
ETG_TUNE=1024 python tools/c1_latency.py LJ-small 2>&1 | grep -v profile
python tools/c1_latency.py LJ-small 2>&1 | grep -v profile
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:expand_warp -s 4 -c 1 -o $O/full_c4_sssp_expand \
   python tools/prof_run.py --config C4 --algs sssp > $O/full_c4.log 2>&1
python tools/ncu_lines.py $O/full_c4_sssp_expand.ncu-rep 30 > $O/full_c4_sssp_expand.lines.txt 2>&1
ncu -i $O/full_c4_sssp_expand.ncu-rep --page raw --csv > $O/full_c4_sssp_expand.raw.csv 2>/dev/null; gzip -f $O/full_c4_sssp_expand.raw.csv
du -sh $O
