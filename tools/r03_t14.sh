#!/bin/bash
sed -n '/cat > \/tmp\/sd.py/,/^PY$/p' tools/r03_sssp_sched.sh > /tmp/mk.sh; bash /tmp/mk.sh
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
python /tmp/sd.py C2 8,10,12,14,16 2>&1
python /tmp/sd.py C3 13,16,18,20,24 2>&1
python /tmp/sd.py C4 5,6,7,8 2>&1
