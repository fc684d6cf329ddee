timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
python tools/e2e_diag.py 0 2>&1 | grep run_host
python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e'])"
