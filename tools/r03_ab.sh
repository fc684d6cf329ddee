#!/bin/bash
# A/B of load-time env switches on the C2 bench (BFS/SSSP/CC per-call ms); args: "NAME=ENV ..." specs
mkdir -p gpurun_out
ab() { tag=$1; shift
  env "$@" python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out gpurun_out/ab_$tag.json > gpurun_out/ab_$tag.log 2>&1
  python -c "import json; d=json.load(open('gpurun_out/ab_$tag.json')); print('$tag', round(d['value'],2), {k:round(v['ms_per_call'],3) for k,v in d['per_alg'].items()}, 'frac', round(d['roofline']['frac'],3), 'scan', round(d['roofline']['scan_share_of_call'],3))" 2>/dev/null || { echo "$tag FAILED"; tail -5 gpurun_out/ab_$tag.log; }
}
for spec in "$@"; do tag=${spec%%:*}; envs=${spec#*:}; ab $tag $envs; done
