#!/bin/bash
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "mid:ETG_X=0" "noahead:ETG_AHEAD_MID=0" "grab2:ETG_TUNE2=1" "old:ETG_AHEAD_MID=0 ETG_TUNE2=1" "mid_b:ETG_X=0"
bash tools/r03_ab.sh "c3mid:ETG_X=0" 2>/dev/null | head -0
for v in "c3_mid:ETG_X=0" "c3_old:ETG_AHEAD_MID=0 ETG_TUNE2=1"; do tag=${v%%:*}; e=${v#*:}
  env $e python bench.py --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out gpurun_out/$tag.json > gpurun_out/$tag.log 2>&1
  python -c "import json; d=json.load(open('gpurun_out/$tag.json')); print('$tag', round(d['value'],2), {k:round(v['ms_per_call'],3) for k,v in d['per_alg'].items()})"
done
