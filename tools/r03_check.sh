#!/bin/bash
# Round-2 re-entry check: full GPU suite + default bench line + smoke
mkdir -p gpurun_out
python -c "import __graft_entry__ as e; e.build(); e.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -x --durations=15 > gpurun_out/gputest.log 2>&1; tail -25 gpurun_out/gputest.log
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 1500 gpurun_out/bench_default.json
