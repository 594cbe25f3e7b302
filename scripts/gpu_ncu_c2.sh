#!/bin/bash
# ncu --set full of one fused C2 step at b = 8192 (row-block chain + the five dW GEMMs); summaries only
mkdir -p gpurun_out/ncuc2; O=gpurun_out/ncuc2
timeout -s KILL 900 ncu --set full --clock-control none -k regex:"rowchain|tc_gemm" -c 6 -f -o $O/c2 \
  python scripts/step_once.py 54,512,512,512,512,7 8192 1 > $O/ncu.log 2>&1; echo "rc=$?"
python scripts/ncu_traffic.py $O/c2.ncu-rep covtype > $O/summary.txt 2>&1; cp profiles/ncu_traffic.json $O/
ncu -i $O/c2.ncu-rep --page details > $O/details.txt 2>&1
rm -f $O/c2.ncu-rep; cat $O/summary.txt | cut -c1-150
