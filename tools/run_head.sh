#!/bin/bash
# Full validation at HEAD (run under gpurun): gpu tests, smoke, bench, ncu launch list.
set -u
OUT=gpurun_out/${1:-head}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.max.sm,clocks.sm --format=csv > $OUT/gpu.csv 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/gpu_tests.txt 2>&1; echo "tests rc=$?"; tail -3 $OUT/gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke.txt
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; tail -1 $OUT/bench.json | cut -c1-600
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_bench.log 2>&1; echo "ncu rc=$?"
