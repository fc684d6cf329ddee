ab() { (cd $1 && python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --json-out /tmp/ab.json > /tmp/ab.log 2>&1; python -c "
import json; d=json.load(open('/tmp/ab.json')); print('$1', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()})"); }
ab _headwt; ab .; ab _headwt; ab .
