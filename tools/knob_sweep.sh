#!/bin/bash
# Sweep K and NO_SMP / NO_UDC on C2 (host loop, launch list per variant). args: "K:flags" ...
for kv in "$@"; do
  K=${kv%%:*}; F=${kv##*:}
  ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"expand|udc_scan" --csv --log-file gpurun_out/knob_${K}_${F}.csv python tools/prof_run.py --algs bfs,sssp,cc --K $K --flags $((32 | F)) > gpurun_out/knob_${K}_${F}.log 2>&1
  echo "== K=$K flags=$F"; python tools/launches.py gpurun_out/knob_${K}_${F}.csv 2>/dev/null | head -4
done
