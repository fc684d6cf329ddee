#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
for v in "dirty1:ETG_X=0" "dirty0:ETG_DIRTY=0"; do tag=${v%%:*}; e=${v#*:}
env $e ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"udc_scan" --csv --log-file gpurun_out/l_$tag.csv python tools/prof_run.py --algs sssp,cc > /dev/null 2>&1
echo "== $tag"; python tools/launches.py gpurun_out/l_$tag.csv 60 2>&1 | head -3; python tools/launches.py gpurun_out/l_$tag.csv 60 2>&1 | tail -27 | awk '{print $1}' | paste -sd' '
done
