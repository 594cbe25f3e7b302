#!/bin/bash
# ncu --set full of the dW GEMMs of a b = 32 C2 step (the layer-0 dW is the step's last kernel)
mkdir -p gpurun_out/small; O=gpurun_out/small
STEPS=3 timeout -s KILL 600 ncu --set full --clock-control none -k regex:tc_gemm_kernel -c 30 -f -o $O/dw \
  python scripts/small_batch_probe.py 32 > $O/ncu2.log 2>&1; echo "rc=$?"
ncu -i $O/dw.ncu-rep --page details > $O/dw_details.txt 2>&1
rm -f $O/dw.ncu-rep
grep -E "tc_gemm_kernel<|  Duration" $O/dw_details.txt | paste - - | sed -E "s/\(CUtensorMap.*\) \(/ (/" | head -30
