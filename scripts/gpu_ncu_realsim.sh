#!/bin/bash
# ncu --set full of one C4 (real-sim-shaped 20958-4096^4-2, b = 8192) mini-batch step's kernels
mkdir -p gpurun_out
timeout -s KILL 900 ncu --set full --clock-control none -k regex:tc_gemm -s 40 -c 13 -o gpurun_out/realsim_full -f \
  python bench.py --config realsim --policy minibatch --steps 1 --warmup 0 --e2e-steps 0 --no-prof --no-cpu-baseline --ttt-epochs 0 > gpurun_out/ncu_realsim.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_realsim.log
