#!/bin/bash
L=$PWD/paper_conf_ipps_wangzlg19_b200
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
bash tools/r03_ab.sh "kr8a:ETG_X=0" "kr6a:ETG_LIB_PATH=$L/libetg_kr6.so" "kr10a:ETG_LIB_PATH=$L/libetg_kr10.so" "kr8b:ETG_X=0" "kr6b:ETG_LIB_PATH=$L/libetg_kr6.so" "kr10b:ETG_LIB_PATH=$L/libetg_kr10.so"
