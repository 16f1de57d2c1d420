#!/bin/bash
# rounding-branch stream priority in the pipelined step (CUALIGN_ROUND_PRIO 0 = highest, 1 = default, 2 = lowest)
set -u
OUT=gpurun_out/prio
mkdir -p $OUT
for rep in 1 2; do
for pr in 0 1 2; do
  CUALIGN_PIPELINE=1 CUALIGN_ROUND_PRIO=$pr timeout 300 python bench.py --no-cpu-baseline --no-e2e > $OUT/b_${pr}_$rep.json 2> $OUT/b_${pr}_$rep.err
  python -c "
import json; d=json.loads(open('$OUT/b_${pr}_$rep.json').read().strip().splitlines()[-1])
print('prio=$pr', round(d['value'],1), d['step_schedule'], {k:round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done; done
