# A/B of expand variants on C2 + sanitizer with the caching allocator off
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
bash tools/ab.sh e1 "ETG_TUNE=0" "ETG_TUNE=1" "ETG_TUNE=131072" "ETG_TUNE=131073" "ETG_TUNE=64" "ETG_TUNE=0" 2>&1
mkdir -p gpurun_out/san
for m in graph hostloop; do
  PYTORCH_NO_CUDA_MEMORY_CACHING=1 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tests/sanitize_run.py $m > gpurun_out/san/memcheck_nocache_$m.txt 2>&1; echo "memcheck $m rc=$?"; tail -3 gpurun_out/san/memcheck_nocache_$m.txt
done
