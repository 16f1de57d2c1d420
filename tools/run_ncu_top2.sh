set -u
OUT=gpurun_out/ncu_top2
mkdir -p $OUT
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-knn --prof-steps 1"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_top2 --launch-skip 30 --launch-count 1 \
   -o $OUT/full_k_top2 python bench.py $ARGS > $OUT/ncu_k_top2.log 2>&1; echo "pipelined rc=$?"
CUALIGN_PIPELINE=2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_top2 --launch-skip 30 --launch-count 1 \
   -o $OUT/full_k_top2_serial python bench.py $ARGS > $OUT/ncu_k_top2_serial.log 2>&1; echo "serial rc=$?"
