python -c "import __graft_entry__ as e; e.build()" > /dev/null 2>&1
L=ETG_LIB_PATH=/root/repo/_ab/libetg
bash tools/ab.sh e10 "${L}_cur.so" "${L}_minb4.so" "${L}_kr10.so" "${L}_kr6.so" "${L}_krw8.so" "${L}_krw4.so" "${L}_cur.so" "${L}_minb4.so" 2>&1
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q 2>&1 | tail -2
