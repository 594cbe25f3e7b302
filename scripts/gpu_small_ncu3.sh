#!/bin/bash
# ncu source-level capture of the layer-0 dW GEMM of a b = 32 C2 step (11th tc_gemm launch)
mkdir -p gpurun_out/small; O=gpurun_out/small
STEPS=3 timeout -s KILL 600 ncu --set full --import-source on --clock-control none -k regex:tc_gemm_kernel --launch-skip 10 --launch-count 1 -f -o $O/dw0 \
  python scripts/small_batch_probe.py 32 > $O/ncu3.log 2>&1; echo "rc=$?"
ncu -i $O/dw0.ncu-rep --page source --csv --print-source sass > $O/dw0_source.csv 2>/dev/null
ncu -i $O/dw0.ncu-rep --page details > $O/dw0_details.txt 2>&1
rm -f $O/dw0.ncu-rep; grep -E "Duration|\(8, 1, 1\)" $O/dw0_details.txt | head -3
