python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
mkdir -p gpurun_out/p1
# SSSP (auto Delta) scans: dense (#4) and moderate (#9); CC scan #1
for sk in 4 9; do
ncu --set full --clock-control none --import-source on -k regex:udc_scan -s $sk -c 1 -o gpurun_out/p1/scan_sssp_$sk \
    python tools/prof_run.py --algs sssp > gpurun_out/p1/scan_sssp_$sk.log 2>&1
python tools/ncu_hot.py gpurun_out/p1/scan_sssp_$sk.ncu-rep 30 > gpurun_out/p1/scan_sssp_$sk.hot.txt 2>&1
done
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan|init_kernel" --csv \
    --log-file gpurun_out/p1/launches_warm.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
run() { echo "== $*"; timeout 300 compute-sanitizer --print-limit 3 "$@" 2>&1 | grep -v "^=========     \|Host Frame\|^=========$" | head -8; }
run --tool memcheck python tools/san_cc.py 32 0 sswp
run --tool synccheck python tools/san_cc.py 32 0 cc
run --tool racecheck python tools/san_cc.py 32 0 cc
run --tool initcheck python tools/san_cc.py 32 0 cc
export ETG_TUNE=16384
run --tool memcheck python tools/san_cc.py 32 0 cc
