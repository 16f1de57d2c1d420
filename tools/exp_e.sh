#!/bin/bash
set -u
OUT=gpurun_out/e_${1:-a}
mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/tests.log 2>&1; echo "tests rc=$? $(tail -1 $OUT/tests.log)"
grep -E "FAIL|Error|error" $OUT/tests.log | head -20
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
python -c "import json; d=json.loads(open('$OUT/bench.json').read().strip().splitlines()[-1]); print(d['value'], d['init_s'], d['e2e']['value'], d['e2e']['align_time_s'], d['kernel_ms_per_step'])"
ARGS="--steps 5 --warmup 3 --no-e2e --no-cpu-baseline --prof-steps 1"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv python bench.py $ARGS > /dev/null 2>&1; echo "launches rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_suitor$' --launch-skip 3 --launch-count 1 -o $OUT/full_k_suitor python bench.py $ARGS > $OUT/ncu_suitor.log 2>&1; echo "ncu suitor rc=$?"
