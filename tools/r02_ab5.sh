python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
B=ETG_LIB_PATH=/root/repo/_ab/libetg_base.so
bash tools/ab.sh e5 "$B" "ETG_TUNE=0" "$B" "ETG_TUNE=0" 2>&1
ncu --metrics gpu__time_duration.sum,l1tex__t_sector_hit_rate.pct,lts__t_requests_srcunit_tex_op_read.sum -k regex:expand_warp -s 3 -c 1 --csv python tools/prof_run.py --algs bfs 2>/dev/null | grep -v "^==" | cut -d, -f13-15
