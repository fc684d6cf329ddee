#!/bin/bash
# A/B bench of engine variants on C2 (short runs, no e2e / cpu baseline); usage: tools/ab.sh tag "ENV=.. ENV2=.." ...
tag=$1; shift
i=0
for envs in "$@"; do
  env $envs python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out gpurun_out/ab_${tag}_$i.json > gpurun_out/ab_${tag}_$i.log 2>&1
  python - "$envs" gpurun_out/ab_${tag}_$i.json <<'PY'
import json, sys
d = json.load(open(sys.argv[2]))
r = d.get("roofline") or {}
print(f"{sys.argv[1]:28s} value {d['value']:7.2f}", {k: (round(v['gteps'], 1), round(v['ms_per_call'], 3)) for k, v in d['per_alg'].items()},
      "frac", round(r.get("frac", 0), 3), "exp", round(r.get("expand_share_of_call", 0), 2), "scan", round(r.get("scan_share_of_call", 0), 2))
PY
  i=$((i+1))
done
