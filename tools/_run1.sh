timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
timeout 300 bash tools/ab.sh live "ETG_TUNE=0|--algs bfs" "ETG_TUNE=2048|--algs bfs" "ETG_TUNE=0|--algs bfs" "ETG_TUNE=2048|--algs bfs"
