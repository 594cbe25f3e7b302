#!/bin/bash
# full GPU suite + C3 / C4 bench lines
mkdir -p gpurun_out/q4; O=gpurun_out/q4
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x --timeout 600 > $O/tests.log 2>&1; tail -3 $O/tests.log
for c in "--config w8a --policy minibatch" "--config w8a" ""; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 $c > $O/b.json 2>$O/b.err
python - "$c" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/q4/b.json").read().strip().splitlines()[-1])
print(sys.argv[1] or "C4", "value", d["value"], "ms", d["ms_per_step"], "tc", d.get("tc_peak_frac"))
for k, v in list(d.get("roofline", {}).get("classes", {}).items())[:12]:
    print("  ", k, v)
PY
done
