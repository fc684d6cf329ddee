#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -3
bash tools/r03_ab.sh "rows4:ETG_SCAN_ROWS=4" "rows0:ETG_SCAN_ROWS=0" "rows1:ETG_SCAN_ROWS=1" "rows8:ETG_SCAN_ROWS=8" "rows16:ETG_SCAN_ROWS=16"
