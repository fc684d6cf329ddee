#!/bin/bash
# compute-sanitizer over the final kernels (host-loop mode; default switches and
# the scan's list/staging paths forced on), summaries -> gpurun_out/san3/
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
O=gpurun_out/san3; mkdir -p $O
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 5 python tests/sanitize_run.py hostloop > $O/${tool}_default.txt 2>&1
  echo "$tool default: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $O/${tool}_default.txt | tail -1) $(grep -c 'ok' $O/${tool}_default.txt) ok-lines"
done
for tool in memcheck racecheck synccheck; do
  ETG_SCAN_LIST=2 ETG_SCAN_ROWS=1 timeout 1200 compute-sanitizer --tool $tool --print-limit 5 python tests/sanitize_run.py hostloop > $O/${tool}_list_staged.txt 2>&1
  echo "$tool list+staged: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' $O/${tool}_list_staged.txt | tail -1) $(grep -c 'ok' $O/${tool}_list_staged.txt) ok-lines"
done
