timeout 900 python -m pytest tests/test_gpu_bench.py -x -q 2>&1 | tail -2
python bench.py --steps 16 --warmup 3 --no-e2e --no-cpu-baseline --no-profile 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], json.dumps(d['per_alg']))"
