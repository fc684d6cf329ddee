#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "lst:ETG_X=0" "lst_b:ETG_X=0" "lst_rows8:ETG_SCAN_ROWS=8"
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"udc_scan" --csv --log-file gpurun_out/l_lst.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
python tools/launches.py gpurun_out/l_lst.csv 80 2>&1 | head -3; python tools/launches.py gpurun_out/l_lst.csv 80 2>&1 | tail -56 | awk '{print $1}' | paste -sd' '
