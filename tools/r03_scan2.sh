#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -3
bash tools/r03_ab.sh "split8:ETG_SPLIT=8" "split1:ETG_SPLIT=1" "split4:ETG_SPLIT=4" "split2:ETG_SPLIT=2"
O=gpurun_out
for idx in 6 11; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:udc_scan -s $idx -c 1 -o $O/scan_sssp_$idx python tools/prof_run.py --config C2 --algs sssp > $O/scan_$idx.log 2>&1
  python tools/ncu_lines.py $O/scan_sssp_$idx.ncu-rep 30 > $O/scan_sssp_$idx.lines.txt 2>&1
  ncu -i $O/scan_sssp_$idx.ncu-rep --page raw --csv > $O/scan_sssp_$idx.raw.csv 2>/dev/null
  python tools/ncu_summary.py $O/scan_sssp_$idx.raw.csv > $O/scan_sssp_$idx.summary.json; cat $O/scan_sssp_$idx.summary.json
  ncu -i $O/scan_sssp_$idx.ncu-rep --page details --csv --section WarpStateStats > $O/scan_sssp_$idx.stall.csv 2>/dev/null
done
