python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
run() { echo "== $*"; timeout 300 compute-sanitizer --tool memcheck --print-limit 3 "$@" 2>&1 | grep -v "^=========     \|Host Frame\|^=========$" | head -12; }
run python tools/san_cc.py 32 0 cc
ETG_TUNE=16384 run python tools/san_cc.py 32 0 cc
run python tools/san_cc.py 32 32 cc
run python tools/san_cc.py 4096 0 cc
run python tools/san_cc.py 32 0 bfs
run python tools/san_cc.py 32 0 sssp
run python tools/san_cc.py 32 2 cc
