#!/bin/bash
mkdir -p gpurun_out/q5; O=gpurun_out/q5
timeout -s KILL 900 python -m pytest tests/test_gpu_head.py tests/test_gpu_step.py -q -x --timeout 300 > $O/tests.log 2>&1; tail -2 $O/tests.log
for c in "--config w8a --policy minibatch" "--config w8a"; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 $c > $O/b.json 2>$O/b.err
python - "$c" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/q5/b.json").read().strip().splitlines()[-1])
print(sys.argv[1] or "C4", "value", d["value"], "ms", d["ms_per_step"], "tc", d.get("tc_peak_frac"))
for k, v in list(d.get("roofline", {}).get("classes", {}).items()):
    if "head" in k or "l3" in k: print("  ", k, v)
PY
done
STEPS=200 timeout -s KILL 300 python scripts/small_batch_probe.py 32,256,1024,2048 2>&1 | tail -4
