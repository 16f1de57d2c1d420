#!/bin/bash
# Suitor launch knobs under the pipelined step (tuned earlier with the rounding alone).
set -u
OUT=gpurun_out/suitorpipe
mkdir -p $OUT
for v in "X=0" "CUALIGN_SUITOR_G=2" "CUALIGN_SUITOR_G=8" "CUALIGN_SUITOR_MINB=16" "CUALIGN_SUITOR_MINB=8" "CUALIGN_SUITOR_PERSIST=1" "X=1"; do
  env $v timeout 300 python bench.py --no-cpu-baseline --no-e2e > $OUT/b_$v.json 2> $OUT/b_$v.err
  python -c "
import json; d=json.loads(open('$OUT/b_$v.json').read().strip().splitlines()[-1])
print('$v', round(d['value'],1), d['step_schedule'], 'match alone', round(d['kernels_isolated']['match']['ms'],4), {k:round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done
