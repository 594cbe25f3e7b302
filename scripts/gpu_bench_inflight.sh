#!/bin/bash
# GPU tests + bench A/B of the host in-flight depth and the fused path (default workload + minibatch)
timeout -s KILL 500 python -m pytest tests -m gpu -q -x --timeout 200 2>&1 | tail -3
for d in 1 2; do for pol in minibatch adaptive; do
  HB_INFLIGHT=$d timeout -s KILL 300 python bench.py --policy $pol --steps 10 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof > gpurun_out/inf_${pol}_$d.json 2>gpurun_out/inf_${pol}_$d.err
  python -c "import json;d=json.loads(open('gpurun_out/inf_${pol}_$d.json').read().strip().splitlines()[-1]);print('inflight=$d $pol', round(d['value']/1e6,2),'M samples/s  e2e',round(d['e2e']['value']/1e6,2), 'tc', round(d['tc_peak_frac'],4))"
done; done
