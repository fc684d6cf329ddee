python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -3
O=gpurun_out/ab3; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
for t in 0 524288 262144; do
  ETG_TUNE=$t timeout 900 python bench.py --config C4 --algs sssp --steps 3 --warmup 2 --no-cpu-baseline --no-e2e --no-profile --json-out $O/c4_$t.json > $O/c4_$t.log 2>&1
  python -c "import json; d=json.load(open('$O/c4_$t.json')); print('C4 tune $t', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()})"
done
bash tools/ab.sh e3 "ETG_TUNE=0" "ETG_TUNE=262144" "ETG_TUNE=0" "ETG_TUNE=262144" 2>&1
