#!/bin/bash
# run-to-run spread of the C2 Adaptive (two workers, Hogwild) bench line: value, calibrated lower
# threshold, update shares
mkdir -p gpurun_out/var; O=gpurun_out/var
for i in 1 2 3 4; do
  timeout 600 python bench.py --config covtype --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof --e2e-steps 0 > $O/b$i.json 2>$O/b$i.err
  python - $i <<'PY'
import json, sys
d = json.loads(open(f"gpurun_out/var/b{sys.argv[1]}.json").read().strip().splitlines()[-1])
print(sys.argv[1], round(d["value"] / 1e6, 2), "M", d["config"]["workers"], d.get("update_share"), d.get("gpu_launches"))
PY
done
