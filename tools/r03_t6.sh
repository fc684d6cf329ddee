#!/bin/bash
for v in "def:ETG_X=0" "nolist:ETG_SCAN_ROWS=0"; do tag=${v%%:*}; e=${v#*:}
env $e ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan" --csv --log-file gpurun_out/l_$tag.csv python tools/prof_run.py --algs sssp > /dev/null 2>&1
echo "== $tag"; python tools/launches.py gpurun_out/l_$tag.csv 60 2>&1 | tail -40 | awk '{print $1}' | paste -sd' '
done
