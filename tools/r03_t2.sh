#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -2
L=$PWD/paper_conf_ipps_wangzlg19_b200
bash tools/r03_ab.sh "main:ETG_X=0" "g4:ETG_LIB_PATH=$L/libetg_g4.so" "g16:ETG_LIB_PATH=$L/libetg_g16.so" "wpw16:ETG_LIB_PATH=$L/libetg_wpw16.so" "main2:ETG_X=0" "rows0:ETG_SCAN_ROWS=0"
python tools/iter_floor.py 2>&1 | grep graph
