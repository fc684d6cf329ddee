#!/bin/bash
L=$PWD/paper_conf_ipps_wangzlg19_b200
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "prev1:ETG_LIB_PATH=$L/libetg_prev.so" "new1:ETG_X=0" "prev2:ETG_LIB_PATH=$L/libetg_prev.so" "new2:ETG_X=0"
