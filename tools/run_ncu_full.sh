#!/bin/bash
# ncu --set full captures of the step's kernels at HEAD (run under gpurun)
set -u
OUT=gpurun_out/${1:-ncu_full}
mkdir -p $OUT
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-knn --prof-steps 1"
for K in k_square_tma k_top2 k_eval k_edge k_suitor; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K --launch-skip 30 --launch-count 1 \
     -o $OUT/full_$K python bench.py $ARGS > $OUT/ncu_$K.log 2>&1; echo "$K rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sbuild_g --launch-count 2 \
   -o $OUT/full_k_sbuild_g python tools/probe_init.py O 1.0 > $OUT/ncu_sbuild.log 2>&1; echo "sbuild rc=$?"
