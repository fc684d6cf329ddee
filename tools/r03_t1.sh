#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -3
bash tools/r03_ab.sh "ticket:ETG_X=0" "ticket_b:ETG_X=1"
python tools/iter_floor.py 2>&1 | grep graph
