#!/bin/bash
# quick GPU iteration: parity tests, short bench, launch list (host-loop mode so ncu sees every kernel)
tag=${1:-q}
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out gpurun_out/bench_$tag.json > gpurun_out/bench_$tag.log 2>&1
python - <<PY
import json
d=json.load(open("gpurun_out/bench_$tag.json"))
r=d["roofline"]
print("value", round(d["value"],2), {k:(round(v["gteps"],1), round(v["ms_per_call"],3)) for k,v in d["per_alg"].items()})
print("roof", round(r["achieved"],1), round(r["frac"],3), {k:round(v["achieved_gbs"],1) for k,v in r["per_alg"].items()}, "expand share", round(r["expand_share_of_call"],3), "scan share", round(r["scan_share_of_call"],3))
PY
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"expand|udc_scan|advance|init_kernel|ctl_begin" --csv --log-file gpurun_out/launches_$tag.csv python tools/prof_run.py --algs bfs,sssp,cc > gpurun_out/launches_$tag.log 2>&1
python tools/launches.py gpurun_out/launches_$tag.csv 2>/dev/null | head -8
