#!/bin/bash
# GPU tests + one bench line with the init phase trace (stderr) -> gpurun_out/<tag>/
set -u
OUT=gpurun_out/${1:-trace}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/gpu_tests.txt 2>&1; echo "tests rc=$?"; tail -2 $OUT/gpu_tests.txt
CUALIGN_INIT_TRACE=1 timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
python - "$OUT/bench.json" <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", d["value"], "ms/step", d["ms_per_step"], "frac", d["roofline"]["frac"])
print("e2e", {k: d["e2e"][k] for k in ("value", "align_time_s")}, "init_s", d.get("init_s"))
print("kernels", d["kernel_ms_per_step"])
PY
grep "\[init\]" $OUT/bench.err | tail -12
