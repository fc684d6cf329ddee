#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
for spec in "sssp 6" "cc 1"; do set -- $spec
timeout 600 ncu --set full --clock-control none --import-source on -k regex:udc_scan -s $2 -c 1 -o $O/sc_$1_$2 python tools/prof_run.py --config C2 --algs $1 > /dev/null 2>&1
python tools/ncu_lines.py $O/sc_$1_$2.ncu-rep 22 > $O/sc_$1_$2.lines.txt 2>&1
ncu -i $O/sc_$1_$2.ncu-rep --page raw --csv > $O/sc_$1_$2.raw.csv 2>/dev/null
python tools/ncu_summary.py $O/sc_$1_$2.raw.csv > $O/sc_$1_$2.summary.json
echo "=== $1 $2"; head -22 $O/sc_$1_$2.lines.txt; head -12 $O/sc_$1_$2.summary.json
python - <<PY
import csv
r=list(csv.reader(open('gpurun_out/sc_$1_$2.raw.csv'))); h,v=r[0],r[2]
out=[]
for i,k in enumerate(h):
    if k.startswith('smsp__pcsamp_warps_issue_stalled') and not k.endswith('not_issued') and v[i] not in ('0',''):
        out.append(k.replace('smsp__pcsamp_warps_issue_stalled_','')+'='+v[i])
    if k in ('smsp__cycles_active.avg','sm__cycles_elapsed.avg'):
        out.append(k+'='+v[i])
print(' '.join(out))
PY
done
