#!/bin/bash
# ncu --set full of the output-layer kernel (and its update kernel) in one C4 step; summaries only
mkdir -p gpurun_out/ncuhead
O=gpurun_out/ncuhead
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"head_" -c 2 -f -o $O/head \
  python scripts/c4_step.py 1 > $O/ncu.log 2>&1; echo "ncu rc=$?"
ncu -i $O/head.ncu-rep --page details > $O/details.txt 2>&1
ncu -i $O/head.ncu-rep --page source --csv --print-source sass -k regex:head_fused > $O/source.csv 2>/dev/null
ls -la $O; rm -f $O/head.ncu-rep
grep -E "Duration|DRAM Throughput|Memory Throughput|Registers|Achieved Occupancy|Block Limit|Warp Cycles|Issue|Stall" $O/details.txt | head -60
