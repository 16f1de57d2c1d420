#!/bin/bash
set -u
OUT=gpurun_out/d_${1:-a}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/tests.log 2>&1; echo "tests rc=$? $(tail -1 $OUT/tests.log)"
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$? $(tail -1 $OUT/smoke.log)"
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; tail -c 600 $OUT/bench.json
timeout 300 python tools/bench_parts.py --pre 300 --n 50 > $OUT/parts.json 2>&1; echo "parts $(tail -1 $OUT/parts.json | cut -c1-330)"
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --prof-steps 1"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv python bench.py $ARGS > /dev/null 2>&1; echo "launches rc=$?"
for K in "k_suitor<:3" "k_eval:3" "k_top2:3"; do
    NAME=${K%%:*}; SKIP=${K##*:}; SAFE=$(echo $NAME | tr -d '<')
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$NAME" \
        --launch-skip $SKIP --launch-count 1 -o $OUT/full_$SAFE python bench.py $ARGS > $OUT/ncu_$SAFE.log 2>&1
    echo "ncu $NAME rc=$?"
done
