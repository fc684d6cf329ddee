#!/bin/bash
sed -n '/cat > \/tmp\/sd.py/,/^PY$/p' tools/r03_sssp_sched.sh > /tmp/mk.sh; bash /tmp/mk.sh
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
python /tmp/sd.py C2 0,6,8,10,12,16 2>&1
ETG_TUNE=8192 python /tmp/sd.py C2 8,12,16,24 2>&1
python /tmp/sd.py C3 0,8,10,13,16 2>&1
