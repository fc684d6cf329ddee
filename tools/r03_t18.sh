#!/bin/bash
L=$PWD/paper_conf_ipps_wangzlg19_b200
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
bash tools/r03_ab.sh "prev1:ETG_LIB_PATH=$L/libetg_prev.so" "new1:ETG_X=0" "prev2:ETG_LIB_PATH=$L/libetg_prev.so" "new2:ETG_X=0" "prev3:ETG_LIB_PATH=$L/libetg_prev.so" "new3:ETG_X=0"
