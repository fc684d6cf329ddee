#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -3
bash tools/r03_ab.sh "list:ETG_X=0" "list2:ETG_X=0"
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan" --csv --log-file gpurun_out/launches_list.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_list.csv 100 2>&1 | head -100
