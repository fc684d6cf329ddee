#!/bin/bash
sed -n '/cat > \/tmp\/sd.py/,/^PY$/p' tools/r03_sssp_sched.sh > /tmp/mk.sh; bash /tmp/mk.sh
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
python /tmp/sd.py C2 10,12,14 2>&1
ETG_TUNE=8192 python /tmp/sd.py C2 12,16,24,32 2>&1
python /tmp/sd.py C3 13,16 2>&1
ETG_TUNE=8192 python /tmp/sd.py C3 16,24,32 2>&1
