#!/bin/bash
L=$PWD/paper_conf_ipps_wangzlg19_b200
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_dist.py -m gpu -q -x 2>&1 | tail -3
bash tools/r03_ab.sh "off1:ETG_DIRTY=0" "on1:ETG_X=0" "off2:ETG_DIRTY=0" "on2:ETG_X=0"
for v in "c3off:ETG_DIRTY=0" "c3on:ETG_X=0"; do tag=${v%%:*}; e=${v#*:}
  env $e python bench.py --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out gpurun_out/$tag.json > gpurun_out/$tag.log 2>&1
  python -c "import json; d=json.load(open('gpurun_out/$tag.json')); print('$tag', round(d['value'],2), {k:round(v['ms_per_call'],3) for k,v in d['per_alg'].items()})"
done
