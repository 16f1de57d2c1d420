#!/bin/bash
set -u
OUT=gpurun_out/exp_dyn_${1:-a}
mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -m gpu -x -q -p no:cacheprovider > $OUT/tests.log 2>&1; echo "tests rc=$? $(tail -1 $OUT/tests.log)"
for V in 6 9; do
  CUALIGN_SQ_VARIANT=$V timeout 300 python tools/bench_parts.py --pre 100 --n 50 > $OUT/parts_$V.json 2> $OUT/parts_$V.err
  python -c "import json; d=json.load(open('$OUT/parts_$V.json')); print('sq var $V', {k: round(v,4) for k,v in d['iterate_ms'].items()}, {k: round(v,4) for k,v in d['round_ms'].items()})"
  CUALIGN_SQ_VARIANT=$V timeout 300 python bench.py --steps 200 --warmup 5 --no-e2e --no-cpu-baseline > $OUT/bench_$V.json 2> $OUT/bench_$V.err
  python -c "import json; d=json.loads(open('$OUT/bench_$V.json').read().strip().splitlines()[-1]); print('bench var $V', round(d['value'],1), {k: round(v,4) for k,v in d['kernel_ms_per_step'].items()})"
done
