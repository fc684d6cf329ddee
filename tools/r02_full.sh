# full GPU test suite + smoke + sanitizer on the shipping (CUDA-graph) path
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
python -c "import __graft_entry__ as e; e.smoke()" 2>&1 | tail -3
timeout 1500 python -m pytest tests -m gpu -q --durations=15 2>&1 | tail -30
mkdir -p gpurun_out/san
timeout 900 compute-sanitizer --tool memcheck python tests/sanitize_run.py graph > gpurun_out/san/memcheck_graph.txt 2>&1; echo "memcheck graph rc=$?"
tail -5 gpurun_out/san/memcheck_graph.txt
