#!/bin/bash
L=$PWD/paper_conf_ipps_wangzlg19_b200
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
bash tools/r03_ab.sh "kr6a:ETG_X=0" "kr4a:ETG_LIB_PATH=$L/libetg_krw4.so" "kr8a:ETG_LIB_PATH=$L/libetg_krw8.so" "kr6b:ETG_X=0" "kr4b:ETG_LIB_PATH=$L/libetg_krw4.so" "kr8b:ETG_LIB_PATH=$L/libetg_krw8.so"
