#!/bin/bash
# Round evidence: full bench line, launch list of one bench step (host loop so ncu sees every
# kernel), and one ncu --set full capture of the dominant kernel (BFS expand, depth 3 of C2).
tag=${1:-r01}
python bench.py --json-out gpurun_out/bench_$tag.json > gpurun_out/bench_$tag.log 2>&1
tail -1 gpurun_out/bench_$tag.log | cut -c1-400
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"expand|udc_scan|init_kernel|ctl_begin|reach" --csv \
    --log-file gpurun_out/launches_$tag.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-profile --flags 32 \
    > gpurun_out/launches_$tag.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:expand_warp -s 3 -c 1 -o gpurun_out/ncu_expand_$tag \
    python tools/prof_run.py --algs bfs > gpurun_out/ncu_expand_$tag.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:expand_warp -s 4 -c 1 -o gpurun_out/ncu_expand_sssp_$tag \
    python tools/prof_run.py --algs sssp > gpurun_out/ncu_expand_sssp_$tag.log 2>&1
ls -la gpurun_out/*$tag*
# warm-cache launch list (no cache flush between kernels: closer to the graph run)
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:"expand|udc_scan|init_kernel|ctl_begin" --csv \
    --log-file gpurun_out/launches_warm_$tag.csv python tools/prof_run.py --algs bfs,sssp,cc > /dev/null 2>&1
python tools/iter_trace.py --algs bfs,sssp,cc --json gpurun_out/trace_$tag.json > gpurun_out/trace_$tag.log 2>&1
