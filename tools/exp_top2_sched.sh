#!/bin/bash
# k_top2 tile width x step schedule (CUALIGN_PIPELINE unset = timed selection, 1 = pipelined, 2 = serial).
set -u
OUT=gpurun_out/top2sched
mkdir -p $OUT
timeout 300 python -m pytest tests/test_gpu_layout.py -x -q > $OUT/tests_layout.txt 2>&1; echo "layout tests rc=$?"; tail -1 $OUT/tests_layout.txt
for tg in 2 1; do
for pipe in auto 1 2 auto; do
  if [ $pipe = auto ]; then unset CUALIGN_PIPELINE; else export CUALIGN_PIPELINE=$pipe; fi
  CUALIGN_TOP2_TG=$tg timeout 300 python bench.py --no-cpu-baseline > $OUT/b_${tg}_$pipe.json 2> $OUT/b_${tg}_$pipe.err
  python -c "
import json; d=json.loads(open('$OUT/b_${tg}_$pipe.json').read().strip().splitlines()[-1])
print('tg=$tg pipe=$pipe', round(d['value'],1), d['step_schedule'], 'e2e', round(d['e2e']['value'],1), d['e2e'].get('schedule'), {k:round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done; done
unset CUALIGN_PIPELINE
