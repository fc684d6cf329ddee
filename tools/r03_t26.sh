#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
ETG_TUNE=8192 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan" --csv --log-file gpurun_out/l_classic16.csv python tools/prof_run.py --algs sssp --sssp-delta 16 > /dev/null 2>&1
python tools/launches.py gpurun_out/l_classic16.csv 120 2>&1 | head -4
