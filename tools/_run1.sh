for i in 1 2 3 4 5; do timeout 300 python -m pytest tests/test_gpu_dist.py -x -q -k "two_processes" 2>&1 | tail -1; done
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
