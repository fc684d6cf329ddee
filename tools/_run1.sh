timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-1500
