#!/bin/bash
# Step-graph overlap experiments (run under gpurun): bench lines for the
# square-pass scheduling / rounding-priority / occupancy knobs.
set -u
OUT=gpurun_out/exp_${1:-overlap}
mkdir -p $OUT
A="--steps 200 --warmup 5 --no-e2e --no-cpu-baseline"
run() { local tag=$1; shift; env "$@" timeout 300 python bench.py $A > $OUT/$tag.json 2> $OUT/$tag.err; echo "$tag rc=$?"; }
run default
run static_occ3 CUALIGN_SQ_VARIANT=7 CUALIGN_SQT_OCC=3
run static_noprio CUALIGN_SQ_VARIANT=7 CUALIGN_ROUND_PRIO=0
run dyn_occ3 CUALIGN_SQT_OCC=3
for f in $OUT/*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1].split('/')[-1], round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'sq', round(d['kernel_ms_per_step']['square'],4), 'match', round(d['kernel_ms_per_step']['match'],4), 'eval', round(d['kernel_ms_per_step']['eval'],4), 'bp_ms', round(d['bp_ms'],4), 'round_ms', round(d['round_ms'],4))
except Exception as e: print(sys.argv[1], 'ERR', e)
PY
done
