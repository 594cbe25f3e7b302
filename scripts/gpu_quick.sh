#!/bin/bash
# Quick GPU check: selected test files (TESTS, default the head kernel + step parity) and one short
# bench line (BENCH_ARGS).
mkdir -p gpurun_out/quick
O=gpurun_out/quick
timeout -s KILL 900 python -m pytest ${TESTS:-tests/test_gpu_head.py tests/test_gpu_step.py} -q -rA --timeout 300 -x -s > $O/tests.log 2>&1
grep -E "passed|failed|Error|assert" $O/tests.log | tail -15
if [ -z "$NO_BENCH" ]; then
timeout -s KILL 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 ${BENCH_ARGS} > $O/bench.json 2> $O/bench.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/quick/bench.json").read().strip().splitlines()[-1])
print("value", d["value"], "ms", d["ms_per_step"], "tc", d.get("tc_peak_frac"), "e2e", d.get("e2e", {}).get("value"))
r = d.get("roofline", {})
print("roofline", r.get("kernel"), r.get("frac"), "kernels_ms", r.get("kernels_ms_per_step"))
for k, v in list(r.get("classes", {}).items())[:20]:
    print("  ", k, v)
PY
tail -3 $O/bench.err
fi
