timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -2
