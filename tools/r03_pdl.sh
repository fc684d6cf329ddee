#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -3
bash tools/r03_ab.sh "pdl1:ETG_PDL=1" "pdl0:ETG_PDL=0" "pdl1b:ETG_PDL=1" "pdl0b:ETG_PDL=0"
python tools/iter_floor.py 2>&1 | tail -5
ETG_PDL=0 python tools/iter_floor.py 2>&1 | tail -5
