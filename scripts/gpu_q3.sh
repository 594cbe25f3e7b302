#!/bin/bash
# head kernel iteration: head tests, C4 + C3 bench lines, ncu of the head kernel in a C4 step
TESTS="tests/test_gpu_head.py" bash scripts/gpu_quick.sh
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --config w8a --policy minibatch > gpurun_out/quick/bench_c3.json 2>gpurun_out/quick/bench_c3.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/quick/bench_c3.json").read().strip().splitlines()[-1])
print("C3 value", d["value"], "ms", d["ms_per_step"], "tc", d.get("tc_peak_frac"))
for k, v in list(d.get("roofline", {}).get("classes", {}).items())[:14]:
    print("  ", k, v)
PY
bash scripts/gpu_ncu_head.sh
STEPS=200 timeout -s KILL 300 python scripts/small_batch_probe.py 32,256,1024,2048 > gpurun_out/quick/small_batch.jsonl 2>&1; cat gpurun_out/quick/small_batch.jsonl | tail -4
