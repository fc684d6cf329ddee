python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
bash tools/ab.sh e4 "ETG_TUNE=0" "ETG_TUNE=1048576" "ETG_TUNE=0" "ETG_TUNE=1048576" 2>&1
for t in 0 1048576; do echo "tune $t"; ETG_TUNE=$t python tools/c1_latency.py C1 2>&1 | grep graph; done
