python -c "import __graft_entry__ as e; e.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -x -q 2>&1 | tail -2
B=ETG_LIB_PATH=/root/repo/_ab/libetg_base.so
bash tools/ab.sh e7 "$B" "ETG_TUNE=0" "$B" "ETG_TUNE=0" 2>&1
python tools/c1_latency.py C1 | grep graph
