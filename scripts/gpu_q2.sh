#!/bin/bash
# quick pass: head + step + hogbatch GPU tests, C4 bench line, C3 mini-batch bench line
TESTS="tests/test_gpu_head.py tests/test_gpu_step.py tests/test_gpu_hogbatch.py" bash scripts/gpu_quick.sh
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --config w8a --policy minibatch > gpurun_out/quick/bench_c3.json 2>gpurun_out/quick/bench_c3.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/quick/bench_c3.json").read().strip().splitlines()[-1])
print("C3 value", d["value"], "ms", d["ms_per_step"], "tc", d.get("tc_peak_frac"))
for k, v in list(d.get("roofline", {}).get("classes", {}).items())[:14]:
    print("  ", k, v)
PY
