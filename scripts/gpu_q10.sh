#!/bin/bash
mkdir -p gpurun_out/q10; O=gpurun_out/q10
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x --timeout 600 > $O/tests.log 2>&1; tail -2 $O/tests.log
for c in "--config covtype --policy minibatch" "--config covtype" "--config w8a --policy minibatch" ""; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof $c > $O/b.json 2>$O/b.err
python - "$c" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/q10/b.json").read().strip().splitlines()[-1])
print(sys.argv[1] or "C4", "value", round(d["value"] / 1e6, 3), "e2e", round(d["e2e"]["value"] / 1e6, 3), "loss", d["e2e"].get("last_train_loss"), "clk", d["clocks"]["sm_mhz"])
PY
done
