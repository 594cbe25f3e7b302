#!/bin/bash
# ncu --set full of the fused chain and of one concurrent dW GEMM at b = 8192 (C2 shape)
mkdir -p gpurun_out
timeout -s KILL 300 ncu --set full --import-source on --clock-control none -k regex:rowchain -s 2 -c 1 \
  -o gpurun_out/rc_full_8192 -f python scripts/rc_one.py 8192 > gpurun_out/ncu_rc.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_rc.log
timeout -s KILL 300 ncu --set full --import-source on --clock-control none -k regex:tc_gemm -s 10 -c 5 \
  -o gpurun_out/dw_full_8192 -f python scripts/rc_one.py 8192 > gpurun_out/ncu_dw.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_dw.log
