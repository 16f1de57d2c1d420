#!/bin/bash
# k_top2 grid cap (blocks per SM, grid-stride tiles) under the pipelined step
set -u
OUT=gpurun_out/top2grid
mkdir -p $OUT
for g in 0 2 4 6 0; do
  CUALIGN_TOP2_GRID=$g timeout 300 python bench.py --no-cpu-baseline --no-e2e > $OUT/b_$g.json 2> $OUT/b_$g.err
  python -c "
import json; d=json.loads(open('$OUT/b_$g.json').read().strip().splitlines()[-1])
print('grid=$g', round(d['value'],1), d['step_schedule'], 'top2 alone', round(d['kernels_isolated']['top2']['ms'],4), {k:round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done
