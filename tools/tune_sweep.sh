#!/bin/bash
# A/B the ETG_TUNE variants on the C2 BFS/SSSP/CC launch lists (host-loop mode)
for t in "$@"; do
  ETG_TUNE=$t ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"expand|udc_scan" --csv --log-file gpurun_out/tune_$t.csv python tools/prof_run.py --algs bfs,sssp,cc > gpurun_out/tune_$t.log 2>&1
  echo "== tune $t"; grep -E "^(bfs|sssp|cc)" gpurun_out/tune_$t.log | sed 's/.vertices_reached.*//' | cut -c1-150
  python tools/launches.py gpurun_out/tune_$t.csv 2>/dev/null | head -4
done
