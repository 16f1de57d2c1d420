#!/bin/bash
set -u
OUT=gpurun_out/c_${1:-a}
mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_knn.py tests/test_gpu_parity.py tests/test_gpu_quality.py -m gpu -x -q -p no:cacheprovider > $OUT/tests.log 2>&1; echo "tests rc=$? $(tail -1 $OUT/tests.log)"
timeout 300 python tools/bench_knn.py > $OUT/knn.jsonl 2> $OUT/knn.err; cat $OUT/knn.jsonl; tail -3 $OUT/knn.err
timeout 300 python tools/bench_parts.py --pre 300 --n 50 > $OUT/parts.json 2>&1; echo "parts $(tail -1 $OUT/parts.json | cut -c1-300)"
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --prof-steps 1"
for K in "k_suitor:3" "k_eval:3" "k_top2:3" "k_edge:3"; do
    NAME=${K%%:*}; SKIP=${K##*:}
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$NAME" \
        --launch-skip $SKIP --launch-count 1 -o $OUT/full_$NAME python bench.py $ARGS > $OUT/ncu_$NAME.log 2>&1
    echo "ncu $NAME rc=$?"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_knn_tc --launch-skip 1 --launch-count 1 \
   -o $OUT/full_k_knn_tc python tools/bench_knn.py --shapes 65536x65536x128x20 --reps 1 > $OUT/ncu_knn.log 2>&1; echo "ncu knn rc=$?"
