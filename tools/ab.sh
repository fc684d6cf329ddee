#!/bin/bash
# A/B bench of engine variants on C2 (short runs, no e2e / cpu baseline).
# usage: tools/ab.sh tag "ENV=.. ENV2=.. [| --bench-arg ...]" ...
tag=$1; shift
i=0
for spec in "$@"; do
  envs=${spec%%|*}
  args=""
  [[ "$spec" == *"|"* ]] && args=${spec#*|}
  env $envs python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $args --json-out gpurun_out/ab_${tag}_$i.json > gpurun_out/ab_${tag}_$i.log 2>&1
  python - "$spec" gpurun_out/ab_${tag}_$i.json <<'PY'
import json, sys
d = json.load(open(sys.argv[2]))
r = d.get("roofline") or {}
print(f"{sys.argv[1]:36s} value {d['value']:7.2f}", {k: (round(v['gteps'], 1), round(v['ms_per_call'], 3)) for k, v in d['per_alg'].items()},
      "frac", round(r.get("frac", 0), 3), "exp", round(r.get("expand_share_of_call", 0), 2), "scan", round(r.get("scan_share_of_call", 0), 2),
      "edges", {k: v.get("edges_processed") for k, v in (r.get("per_alg") or {}).items()})
PY
  i=$((i+1))
done
