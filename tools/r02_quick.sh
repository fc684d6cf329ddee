set -x
nvidia-smi --query-gpu=name,memory.total --format=csv; free -g | head -2; nproc
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
python -c "import __graft_entry__ as e; e.smoke()" 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_dist.py tests/test_gpu_parity.py -x -q 2>&1 | tail -15
timeout 300 python bench.py --gpus 2 --steps 3 --warmup 3 --no-e2e 2>&1 | tail -3
timeout 300 python bench.py --gpus 2 --steps 3 --warmup 3 --push 2>&1 | tail -3
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/repro tools/sanitize_graph_repro.cu && /tmp/repro && timeout 300 compute-sanitizer --tool memcheck /tmp/repro 2>&1 | tail -8
