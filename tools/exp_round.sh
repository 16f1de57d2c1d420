#!/bin/bash
# Rounding (a7+a8) diagnostics at a fixed BP state (run under gpurun):
# per-kernel times of round-only graph replays for Suitor register caps /
# tile widths, and the Suitor scan / proposal statistics of one un-captured round.
set -u
OUT=gpurun_out/exp_round_${1:-a}
mkdir -p $OUT
for V in "MINB=0" "MINB=10" "MINB=12" "MINB=16" "G=8" "G=2"; do
  env CUALIGN_SUITOR_$V timeout 300 python tools/bench_parts.py --pre 300 --n 50 > $OUT/parts_$V.json 2> $OUT/parts_$V.err
  python -c "import json; d=json.load(open('$OUT/parts_$V.json')); print('$V', {k: round(v,4) for k,v in d['round_ms'].items()})"
done
CUALIGN_MATCH_DEBUG=1 timeout 300 python tools/probe_suitor.py > $OUT/probe.log 2>&1
grep suitor $OUT/probe.log | tail -12
