timeout 900 python -m pytest tests/test_gpu_full.py -x -q -k push 2>&1 | tail -5
python bench.py --partitioned --push auto --algs sssp,cc --steps 5 --warmup 3 2>&1 | tail -1
python bench.py --partitioned --algs sssp,cc --steps 5 --warmup 3 2>&1 | tail -1
