#!/bin/bash
# k_edge variants (EPT x register cap) at a fixed BP state (run under gpurun)
set -u
OUT=gpurun_out/exp_edge_${1:-a}
mkdir -p $OUT
for V in 0 1 2 3 4 5; do
  CUALIGN_EDGE_VAR=$V timeout 300 python tools/bench_parts.py --pre 100 --n 50 > $OUT/parts_$V.json 2> $OUT/parts_$V.err
  python -c "import json; d=json.load(open('$OUT/parts_$V.json')); print('edge var $V', {k: round(v,4) for k,v in d['iterate_ms'].items()})"
done
