#!/bin/bash
# per-kernel device times of small-batch C2 steps (b = 32): ncu launch list of the probe
mkdir -p gpurun_out/small; O=gpurun_out/small
STEPS=20 timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_b32.csv \
  python scripts/small_batch_probe.py 32 > $O/ncu.log 2>&1; echo "rc=$?"
python scripts/launches.py $O/launches_b32.csv | tail -20
