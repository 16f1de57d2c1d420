#!/bin/bash
# ncu captures + atomic-free square probe (run under gpurun)
set -u
OUT=gpurun_out/prof_${1:-b}
mkdir -p $OUT
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --prof-steps 1"
for V in 6 8; do
  CUALIGN_SQ_VARIANT=$V timeout 300 python tools/bench_parts.py --pre 50 --n 30 > $OUT/parts_v$V.json 2>&1; echo "v$V $(tail -1 $OUT/parts_v$V.json | cut -c1-400)"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_square_tma --launch-skip 4 --launch-count 1 \
   -o $OUT/full_k_square_tma python bench.py $ARGS > $OUT/ncu_sq.log 2>&1; echo "ncu sq rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_knn_tc --launch-skip 1 --launch-count 1 \
   -o $OUT/full_k_knn_tc python tools/bench_knn.py --shapes 65536x65536x128x20 --reps 1 > $OUT/ncu_knn.log 2>&1; echo "ncu knn rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/knn_launches.csv \
   python tools/bench_knn.py --shapes 200000x200000x128x20 --reps 1 > /dev/null 2>&1; echo "ncu knn list rc=$?"
