#!/bin/bash
L=$PWD/paper_conf_ipps_wangzlg19_b200
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -2
bash tools/r03_ab.sh "prev1:ETG_LIB_PATH=$L/libetg_prev.so" "defer1:ETG_X=0" "aheadall1:ETG_TUNE=32768" "prev2:ETG_LIB_PATH=$L/libetg_prev.so" "defer2:ETG_X=0" "aheadall2:ETG_TUNE=32768"
for v in "c3prev:ETG_LIB_PATH=$L/libetg_prev.so" "c3defer:ETG_X=0" "c3all:ETG_TUNE=32768"; do tag=${v%%:*}; e=${v#*:}
  env $e python bench.py --config C3 --algs bfs,sssp --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out gpurun_out/$tag.json > gpurun_out/$tag.log 2>&1
  python -c "import json; d=json.load(open('gpurun_out/$tag.json')); print('$tag', round(d['value'],2), {k:round(v['ms_per_call'],3) for k,v in d['per_alg'].items()})"
done
