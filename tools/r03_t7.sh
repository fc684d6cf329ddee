#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
timeout 600 env ETG_SCAN_LIST=2 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "list1:ETG_SCAN_LIST=1" "list2:ETG_SCAN_LIST=2" "list1b:ETG_SCAN_LIST=1" "list2b:ETG_SCAN_LIST=2"
for v in "l1:ETG_SCAN_LIST=1" "l2:ETG_SCAN_LIST=2"; do tag=${v%%:*}; e=${v#*:}
env $e ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"udc_scan" --csv --log-file gpurun_out/l_$tag.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
echo "== $tag"; python tools/launches.py gpurun_out/l_$tag.csv 80 2>&1 | tail -56 | awk '{print $1}' | paste -sd' '
done
