#!/bin/bash
# Rounding (a7+a8) diagnostics at a fixed BP state (run under gpurun):
# per-kernel times of round-only graph replays for Suitor tile widths, and
# the Suitor scan / proposal statistics of one un-captured round.
set -u
OUT=gpurun_out/exp_round_${1:-a}
mkdir -p $OUT
for G in 0 2 4 8 16; do
  CUALIGN_SUITOR_G=$G timeout 300 python tools/bench_parts.py --pre 300 --n 50 > $OUT/parts_G$G.json 2> $OUT/parts_G$G.err
  echo "G=$G $(cat $OUT/parts_G$G.json)"
done
CUALIGN_MATCH_DEBUG=1 timeout 300 python tools/probe_suitor.py > $OUT/probe.log 2>&1
tail -20 $OUT/probe.log
