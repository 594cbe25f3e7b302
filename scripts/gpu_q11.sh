#!/bin/bash
mkdir -p gpurun_out/q11; O=gpurun_out/q11
timeout -s KILL 900 python -m pytest tests/test_gpu_hogbatch.py -q -x --timeout 300 > $O/tests.log 2>&1; tail -2 $O/tests.log
for rep in 1 2; do for c in "" "--config w8a --policy minibatch"; do
timeout 600 python bench.py --steps 8 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof $c > $O/b.json 2>$O/b.err
python - "$c" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/q11/b.json").read().strip().splitlines()[-1])
print(sys.argv[1] or "C4", "value", round(d["value"] / 1e6, 3), "e2e", round(d["e2e"]["value"] / 1e6, 3), "gap %.1f%%" % (100 * (1 - d["e2e"]["value"] / d["value"])), "clk", d["clocks"]["sm_mhz"])
PY
done; done
