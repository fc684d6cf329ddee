timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "auto or near_far or wave" 2>&1 | tail -2
for c in C2 C3; do timeout 600 python bench.py --config $c --algs sssp --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-profile --json-out /tmp/x.json > /tmp/x.log 2>&1; python -c "
import json; d=json.load(open('/tmp/x.json')); print('$c auto', round(d['value'],2), round(d['per_alg']['sssp']['ms_per_call'],3))"; done
timeout 600 python bench.py --config C4 --algs sssp --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --no-profile --json-out /tmp/x.json > /tmp/x.log 2>&1; python -c "
import json; d=json.load(open('/tmp/x.json')); print('C4 auto', round(d['value'],2), round(d['per_alg']['sssp']['ms_per_call'],3))"
