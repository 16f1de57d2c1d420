#!/bin/bash
# A/B of the working tree's library against lib/old (run under gpurun)
set -u
OUT=gpurun_out/ab_${1:-a}
mkdir -p $OUT
OLD=$PWD/paper_conf_sc_xiangkfah23_b200/lib/old/libcualign_bp.so
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/tests.log 2>&1; echo "tests rc=$? $(tail -1 $OUT/tests.log)"
timeout 300 python tools/bench_knn.py > $OUT/knn_new.jsonl 2> $OUT/knn_new.err; echo knn_new; cat $OUT/knn_new.jsonl
CUALIGN_LIB=$OLD timeout 300 python tools/bench_knn.py > $OUT/knn_old.jsonl 2> $OUT/knn_old.err; echo knn_old; cat $OUT/knn_old.jsonl
A="--steps 200 --warmup 5 --no-e2e --no-cpu-baseline"
for v in new old; do
  if [ $v = old ]; then export CUALIGN_LIB=$OLD; else unset CUALIGN_LIB; fi
  timeout 300 python bench.py $A > $OUT/bench_$v.json 2> $OUT/bench_$v.err
  python -c "import json,sys; d=json.loads(open('$OUT/bench_$v.json').read().strip().splitlines()[-1]); print('$v', round(d['value'],1), d['kernel_ms_per_step'])"
  timeout 300 python tools/bench_parts.py --pre 300 --n 50 > $OUT/parts_$v.json 2> $OUT/parts_$v.err; echo "parts_$v $(cat $OUT/parts_$v.json)"
done
unset CUALIGN_LIB
