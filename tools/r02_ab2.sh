python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py -x -q 2>&1 | tail -2
B=ETG_LIB_PATH=/root/repo/_ab/libetg_base.so
bash tools/ab.sh e2 "$B" "ETG_TUNE=0" "$B" "ETG_TUNE=0" 2>&1
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
timeout 300 compute-sanitizer --tool synccheck --print-limit 4 python tools/san_cc.py 32 0 cc 2>&1 | head -60
