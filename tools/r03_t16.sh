#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" 2>&1 | tail -1
timeout 600 env ETG_TUNE=4194304 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "c1_all or golden or other_shapes" 2>&1 | tail -2
bash tools/r03_ab.sh "base:ETG_X=0" "cclive:ETG_TUNE=4194304" "base2:ETG_X=0" "cclive2:ETG_TUNE=4194304"
