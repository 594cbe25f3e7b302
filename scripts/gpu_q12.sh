#!/bin/bash
# e2e gap probe: staging in one chunk (no densify kernels concurrent with training) vs default chunks
mkdir -p gpurun_out/q12; O=gpurun_out/q12
for c in "" "--config w8a --policy minibatch"; do for opt in "" "--opt stage_rows=1000000"; do
timeout 600 python bench.py --steps 8 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof $c $opt > $O/b.json 2>$O/b.err
python - "$c $opt" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/q12/b.json").read().strip().splitlines()[-1])
print(sys.argv[1] or "C4", "value", round(d["value"] / 1e6, 3), "e2e", round(d["e2e"]["value"] / 1e6, 3), "gap %.1f%%" % (100 * (1 - d["e2e"]["value"] / d["value"])), "clk", d["clocks"]["sm_mhz"])
PY
done; done
