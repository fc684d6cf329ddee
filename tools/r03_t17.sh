#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "trim:ETG_X=0" "trim2:ETG_X=0"
