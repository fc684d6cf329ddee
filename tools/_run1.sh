python tools/persist_diag.py --tunes 0,1024,prof 2>&1 | grep -v Warn
ETG_LIB_PATH=paper_conf_ipps_wangzlg19_b200/libetg_sleep.so python tools/persist_diag.py --tunes 0 2>&1 | grep -v Warn
