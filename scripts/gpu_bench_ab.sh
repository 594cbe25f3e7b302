#!/bin/bash
# A/B of the step implementations on the default workload (no oracle baseline / TTT)
mkdir -p gpurun_out
for rc in 1 0; do
  for pol in minibatch adaptive; do
    HB_ROWCHAIN=$rc timeout -s KILL 300 python bench.py --policy $pol --steps 10 --warmup 3 --no-cpu-baseline --ttt-epochs 0 \
      > gpurun_out/ab_${pol}_rc${rc}.json 2> gpurun_out/ab_${pol}_rc${rc}.err
    echo "rc=$rc $pol exit=$?"
  done
done
