ab() { (env $1 python bench.py --steps $3 --warmup 1 --no-e2e --no-cpu-baseline --no-profile --algs sssp --config $2 --json-out /tmp/ab.json > /tmp/ab.log 2>&1; python -c "
import json; d=json.load(open('/tmp/ab.json')); print('$1 $2', round(d['value'],2), {k:(round(v['gteps'],1), round(v['ms_per_call'],3)) for k,v in d['per_alg'].items()})"); }
ab ETG_TUNE=0 C4 3; ab ETG_LIB_PATH=paper_conf_ipps_wangzlg19_b200/libetg_shs.so C4 3
ab ETG_TUNE=0 C3 10; ab ETG_LIB_PATH=paper_conf_ipps_wangzlg19_b200/libetg_shs.so C3 10
ab ETG_TUNE=0 C2 10; ab ETG_LIB_PATH=paper_conf_ipps_wangzlg19_b200/libetg_shs.so C2 10
