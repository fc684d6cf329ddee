#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
for idx in 3 9; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:expand_warp -s $idx -c 1 -o $O/exp_sssp_$idx python tools/prof_run.py --config C2 --algs sssp > /dev/null 2>&1
python tools/ncu_lines.py $O/exp_sssp_$idx.ncu-rep 25 > $O/exp_sssp_$idx.lines.txt 2>&1
ncu -i $O/exp_sssp_$idx.ncu-rep --page raw --csv > $O/exp_sssp_$idx.raw.csv 2>/dev/null
python tools/ncu_summary.py $O/exp_sssp_$idx.raw.csv > $O/exp_sssp_$idx.summary.json
echo "=== $idx"; head -25 $O/exp_sssp_$idx.lines.txt; cat $O/exp_sssp_$idx.summary.json | head -14
python - <<PY
import csv
r=list(csv.reader(open('gpurun_out/exp_sssp_$idx.raw.csv'))); h,v=r[0],r[2]
for i,k in enumerate(h):
    if k.startswith('smsp__pcsamp_warps_issue_stalled') and not k.endswith('not_issued') and v[i] not in ('0',''):
        print(k.replace('smsp__pcsamp_warps_issue_stalled_',''), v[i])
    if k in ('smsp__cycles_active.avg','sm__cycles_elapsed.avg'):
        print(k, v[i])
PY
done
