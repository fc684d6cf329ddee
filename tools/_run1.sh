timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
ab() { (cd $1 && env $2 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $3 --json-out /tmp/ab.json > /tmp/ab.log 2>&1; python -c "
import json; d=json.load(open('/tmp/ab.json')); print('$1 $2', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()})"); }
ab . ETG_TUNE=0; ab . ETG_TUNE=0
