for dl in 3 4 8; do timeout 600 python bench.py --config C4 --algs sssp --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-profile --sssp-delta $dl --json-out /tmp/c4.json > /tmp/c4.log 2>&1; python -c "
import json; d=json.load(open('/tmp/c4.json')); print('C4 delta $dl', round(d['value'],2), round(d['per_alg']['sssp']['ms_per_call'],3))"; done
