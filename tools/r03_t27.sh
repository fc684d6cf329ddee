#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -3
sed -n '/cat > \/tmp\/sd.py/,/^PY$/p' tools/r03_sssp_sched.sh > /tmp/mk.sh; bash /tmp/mk.sh
python /tmp/sd.py C2 12 2>&1
ETG_TUNE=8192 python /tmp/sd.py C2 8,12,16,24 2>&1
python /tmp/sd.py C3 13 2>&1
ETG_TUNE=8192 python /tmp/sd.py C3 16,24,32 2>&1
bash tools/r03_ab.sh "wave:ETG_X=0"
