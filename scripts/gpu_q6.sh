#!/bin/bash
# hogbatch / staging tests + the C4 bench line (device value and e2e)
mkdir -p gpurun_out/q6; O=gpurun_out/q6
timeout -s KILL 900 python -m pytest tests/test_gpu_hogbatch.py -q -x --timeout 300 > $O/tests.log 2>&1; tail -2 $O/tests.log
timeout 600 python bench.py --steps 8 --warmup 3 --no-cpu-baseline --ttt-epochs 0 > $O/b.json 2>$O/b.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/q6/b.json").read().strip().splitlines()[-1])
print("C4 value", d["value"], "ms", d["ms_per_step"], "tc", d.get("tc_peak_frac"), "e2e", d["e2e"], "clk", d["clocks"])
PY
