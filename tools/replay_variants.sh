#!/bin/bash
# replay C2 BFS depth 3/4 (and SSSP 4) with each prebuilt library variant in build/
python tools/replay.py --tunes 0,32,16 2>&1 | sed 's/^/[default] /'
for so in build/libetg_*.so; do
  ETG_LIB_PATH=$so python tools/replay.py --tunes 0 2>&1 | sed "s|^|[$(basename $so)] |"
done
python tools/replay.py --alg sssp --depths 4 --tunes 0 2>&1 | sed 's/^/[default] /'
