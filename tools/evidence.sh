#!/bin/bash
# Round evidence sweep: every config at 1 GPU and the ablations.  Each line -> gpurun_out/ev_<name>.json
run() { name=$1; shift; timeout ${T:-300} python bench.py --no-e2e --no-cpu-baseline --no-profile --json-out gpurun_out/ev_$name.json "$@" > gpurun_out/ev_$name.log 2>&1; \
  python -c "import json; d=json.load(open('gpurun_out/ev_$name.json')); print('$name', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()})" 2>/dev/null || echo "$name FAILED"; }
run c1 --config C1 --steps 20 --warmup 5
run c2_default --steps 10 --warmup 3
run c2_nosmp --steps 10 --warmup 3 --flags 4
run c2_smpshared --steps 10 --warmup 3 --flags 128
run c2_noudc --steps 10 --warmup 3 --flags 2
run c2_k8 --steps 10 --warmup 3 --K 8
run c2_k16 --steps 10 --warmup 3 --K 16
run c2_k64 --steps 10 --warmup 3 --K 64
run c2_k256 --steps 10 --warmup 3 --K 256
run c2_hostloop --steps 10 --warmup 3 --flags 32
run c2_sssp_paper --algs sssp --steps 10 --warmup 3 --sssp-delta 0
run c2_sssp_wave8 --algs sssp --steps 10 --warmup 3 --sssp-delta 8
run c2_sssp_wave16 --algs sssp --steps 10 --warmup 3 --sssp-delta 16
ETG_TUNE=8192 run c2_sssp_classic16 --algs sssp --steps 10 --warmup 3 --sssp-delta 16
run c2_hostedges --algs bfs,sssp --steps 3 --warmup 1 --host-edges
run c3_udc --config C3 --algs bfs,sssp --steps 10 --warmup 3
run c3_sssp_paper --config C3 --algs sssp --steps 10 --warmup 3 --sssp-delta 0
run c3_noudc --config C3 --algs bfs,sssp --steps 10 --warmup 3 --flags 2
T=600 run c4_sssp --config C4 --algs sssp --steps 3 --warmup 1
T=600 run c4_sssp_paper --config C4 --algs sssp --steps 3 --warmup 1 --sssp-delta 0
T=600 run c4_sssp_noudc --config C4 --algs sssp --steps 2 --warmup 1 --flags 2
T=600 run c5_bfs --config C5 --algs bfs --steps 3 --warmup 1
