#!/bin/bash
# Round profiling on one GPU (run under gpurun): bench line, launch list, one
# ncu --set full capture per hot kernel.  Outputs in gpurun_out/prof_<tag>/.
set -u
TAG=${1:-r01}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --prof-steps 1"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > $OUT/gpu.csv
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py $ARGS > /dev/null 2>&1
for K in "k_square:4" "k_edge:3" "k_top2:3" "k_suitor<:3" "k_eval:3"; do
    NAME=${K%%:*}; SKIP=${K##*:}
    SAFE=$(echo $NAME | tr -d '<')
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$NAME" \
        --launch-skip $SKIP --launch-count 1 -o $OUT/full_$SAFE python bench.py $ARGS > $OUT/ncu_$SAFE.log 2>&1
done
echo done
