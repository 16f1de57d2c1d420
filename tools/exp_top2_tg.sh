#!/bin/bash
# k_top2 tile-width experiment (CUALIGN_TOP2_TG = 8 / 4 / 2): parity tests and bench per width.
set -u
OUT=gpurun_out/top2tg
mkdir -p $OUT
for tg in 1; do
  CUALIGN_TOP2_TG=$tg timeout 600 python -m pytest tests -m gpu -x -q > $OUT/tests_$tg.txt 2>&1; echo "tests tg=$tg rc=$?"; tail -1 $OUT/tests_$tg.txt
done
for rep in 1 2; do
for tg in 4 2 1; do
  CUALIGN_TOP2_TG=$tg timeout 300 python bench.py --no-e2e --no-cpu-baseline > $OUT/bench_${tg}_$rep.json 2> $OUT/bench_${tg}_$rep.err
  python -c "
import json,sys; d=json.loads(open('$OUT/bench_${tg}_$rep.json').read().strip().splitlines()[-1])
print('tg=$tg', round(d['value'],1), 'top2', d['kernels_isolated']['top2'], 'step top2', d['kernel_ms_per_step']['top2'])"
done; done
