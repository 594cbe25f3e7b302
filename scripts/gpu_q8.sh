#!/bin/bash
# staging changes: hogbatch tests + e2e of C4 / C3 / C2 mini-batch
mkdir -p gpurun_out/q8; O=gpurun_out/q8
timeout -s KILL 900 python -m pytest tests/test_gpu_hogbatch.py tests/test_gpu_multi.py -q -x --timeout 300 > $O/tests.log 2>&1; tail -2 $O/tests.log
for c in "" "--config w8a --policy minibatch" "--config covtype --policy minibatch"; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof $c > $O/b.json 2>$O/b.err
python - "$c" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/q8/b.json").read().strip().splitlines()[-1])
print(sys.argv[1] or "C4", "value", round(d["value"] / 1e6, 3), "e2e", round(d["e2e"]["value"] / 1e6, 3), "clk", d["clocks"]["sm_mhz"])
PY
done
