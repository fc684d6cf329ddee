# Round-2 evidence: bench lines with roofline for every config, expand traffic of
# the same launches, Fig. 7 analogue on C3, ncu --set full of the C4 / C5 dominant
# expand launch and of a dense / sparse scan.
set -u
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
O=gpurun_out/ev2; mkdir -p $O
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
# 1. expand traffic of one call per algorithm (host loop: every launch visible to ncu)
tr() { cfg=$1; algs=$2; tag=${cfg}_${algs//,/+}
  timeout 1200 ncu --metrics $M --cache-control none --clock-control none -k regex:expand_warp --csv \
    --log-file $O/traffic_$tag.csv python tools/prof_run.py --config $cfg --algs $algs --json $O/traffic_$tag.stats.json > $O/traffic_$tag.log 2>&1
  python tools/traffic_summary.py $O/traffic_$tag.csv $O/traffic_$tag.stats.json > $O/expand_traffic_$tag.json && \
    python -c "import json;d=json.load(open('$O/expand_traffic_$tag.json'));print('$tag', d['launches'], round(d['dram_over_alg'],2), round(d['alg_gbs_under_ncu']), round(d['dram_gbs_under_ncu']))"
  gzip -f $O/traffic_$tag.csv; }
tr C2 bfs,sssp,cc
tr C3 bfs,sssp
tr C4 sssp
tr C5 bfs
mkdir -p profiles/r02 && cp $O/expand_traffic_*.json profiles/r02/
# 2. bench lines (roofline on) for every config
b() { name=$1; shift; timeout ${T:-900} python bench.py --json-out $O/bench_$name.json "$@" > $O/bench_$name.log 2>&1; \
  python -c "import json; d=json.load(open('$O/bench_$name.json')); r=d['roofline'] or {}; print('$name', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()}, 'frac', round(r.get('frac',0),3), 'traffic', r.get('traffic'))" 2>/dev/null || { echo "$name FAILED"; tail -5 $O/bench_$name.log; }; }
b c2
b c3 --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-cpu-baseline
T=1500 b c4 --config C4 --algs sssp --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
T=1500 b c5 --config C5 --algs bfs --steps 3 --warmup 3 --no-cpu-baseline --no-e2e
b c1 --config C1 --steps 20 --warmup 5 --no-e2e
# 3. Fig. 7 analogue on C3 (Sec. VI-C): SMP look-ahead (default) / shared-memory TMA stages / off
F=gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active
for v in "0 lookahead" "128 smpshared" "4 nosmp"; do set -- $v
  timeout 900 ncu --metrics $F --cache-control none --clock-control none -k regex:expand_warp --csv \
    --log-file $O/fig7_$2.csv python tools/prof_run.py --config C3 --algs bfs,sssp --flags $((32 | $1)) > $O/fig7_$2.log 2>&1
  python tools/ncu_agg.py $O/fig7_$2.csv expand > $O/fig7_$2.json; echo "fig7 $2"; head -14 $O/fig7_$2.json; gzip -f $O/fig7_$2.csv
done
# 4. ncu --set full: dominant expand launch of C4 SSSP and C5 BFS, C2 SSSP scans (dense #4, sparse #15)
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:expand_warp -s 4 -c 1 -o $O/full_c4_sssp_expand \
   python tools/prof_run.py --config C4 --algs sssp > $O/full_c4.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:expand_warp -s 3 -c 1 -o $O/full_c5_bfs_expand \
   python tools/prof_run.py --config C5 --algs bfs > $O/full_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:udc_scan -s 15 -c 1 -o $O/full_c2_sssp_scan15 \
   python tools/prof_run.py --config C2 --algs sssp > $O/full_scan15.log 2>&1
for r in $O/*.ncu-rep; do python tools/ncu_lines.py $r 30 > ${r%.ncu-rep}.lines.txt 2>&1
  ncu -i $r --page raw --csv > ${r%.ncu-rep}.raw.csv 2>/dev/null; gzip -f ${r%.ncu-rep}.raw.csv; done
du -sh $O; ls -la $O
# keep the pull under 64 MiB: drop the biggest reports if needed
while [ $(du -sm gpurun_out | cut -f1) -gt 60 ]; do big=$(ls -S $O/*.ncu-rep 2>/dev/null | head -1); [ -z "$big" ] && break; echo "dropping $big"; rm -f $big; done
