#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 env ETG_TUNE=2097152 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_big.py -m gpu -q -x -k c4 2>&1 | tail -2
for v in "c4_16:ETG_X=0" "c4_32:ETG_TUNE=1048576"; do tag=${v%%:*}; e=${v#*:}
  env $e timeout 900 python bench.py --config C4 --algs sssp --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --json-out gpurun_out/$tag.json > gpurun_out/$tag.log 2>&1
  python -c "import json; d=json.load(open('gpurun_out/$tag.json')); print('$tag', round(d['value'],2), {k:round(v['ms_per_call'],3) for k,v in d['per_alg'].items()}, 'frac', round(d['roofline']['frac'],3))" || tail -3 gpurun_out/$tag.log
done
