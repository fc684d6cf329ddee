#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:udc_scan -s 0 -c 1 -o $O/scan_cc0 python tools/prof_run.py --config C2 --algs cc > /dev/null 2>&1
python tools/ncu_lines.py $O/scan_cc0.ncu-rep 30 > $O/scan_cc0.lines.txt 2>&1
ncu -i $O/scan_cc0.ncu-rep --page raw --csv > $O/scan_cc0.raw.csv 2>/dev/null
python tools/ncu_summary.py $O/scan_cc0.raw.csv > $O/scan_cc0.summary.json
head -30 $O/scan_cc0.lines.txt; cat $O/scan_cc0.summary.json
python - <<'PY'
import csv
r=list(csv.reader(open('gpurun_out/scan_cc0.raw.csv'))); h,v=r[0],r[2]
for i,k in enumerate(h):
    if k.startswith('smsp__pcsamp_warps_issue_stalled') and not k.endswith('not_issued') and v[i] not in ('0',''):
        print(k.replace('smsp__pcsamp_warps_issue_stalled_',''), v[i])
    if k in ('dram__throughput.avg.pct_of_peak_sustained_elapsed','smsp__cycles_active.avg','sm__cycles_elapsed.avg','l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum','smsp__thread_inst_executed_per_inst_executed.ratio'):
        print(k, v[i])
PY
