#!/bin/bash
# square pass: static chunk stride (CUALIGN_SQ_DYN=0) vs chunk queue (1); parity suite under the queue first.
set -u
OUT=gpurun_out/sqdyn
mkdir -p $OUT
CUALIGN_SQ_DYN=1 timeout 400 python -m pytest tests -m gpu -x -q > $OUT/tests_dyn.txt 2>&1; echo "tests dyn rc=$?"; tail -1 $OUT/tests_dyn.txt
for rep in 1 2; do
for dyn in 0 1; do
  CUALIGN_SQ_DYN=$dyn timeout 300 python bench.py --no-cpu-baseline > $OUT/b_${dyn}_$rep.json 2> $OUT/b_${dyn}_$rep.err
  python -c "
import json; d=json.loads(open('$OUT/b_${dyn}_$rep.json').read().strip().splitlines()[-1])
print('dyn=$dyn', round(d['value'],1), d['step_schedule'], 'e2e', round(d['e2e']['value'],1), 'sq alone', round(d['kernels_isolated']['square']['ms'],4), {k:round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done; done
