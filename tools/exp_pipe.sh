#!/bin/bash
# step pipeline x square scheduling (run under gpurun)
set -u
OUT=gpurun_out/exp_pipe_${1:-a}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/tests.log 2>&1; echo "tests rc=$? $(tail -1 $OUT/tests.log)"
for V in "P1_S6:CUALIGN_PIPELINE=1 CUALIGN_SQ_VARIANT=6" "P0_S6:CUALIGN_PIPELINE=0 CUALIGN_SQ_VARIANT=6" "P1_S9:CUALIGN_PIPELINE=1 CUALIGN_SQ_VARIANT=9" "P0_S9:CUALIGN_PIPELINE=0 CUALIGN_SQ_VARIANT=9"; do
  TAG=${V%%:*}; ENVS=${V#*:}
  env $ENVS timeout 300 python bench.py --steps 200 --warmup 5 --no-e2e --no-cpu-baseline > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
  python -c "import json; d=json.loads(open('$OUT/bench_$TAG.json').read().strip().splitlines()[-1]); print('$TAG', round(d['value'],1), d['best_score'], {k: round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done
