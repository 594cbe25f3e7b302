#!/bin/bash
for cfg in "0 4" "64 4" "128 4" "256 4" "128 8" "256 8" "256 2"; do
  set -- $cfg
  echo "== HB_WGRAD_BN=$1 HB_MAX_SPLITS=$2"
  HB_WGRAD_BN=$1 HB_MAX_SPLITS=$2 timeout -s KILL 60 python scripts/gemm_bench.py 2,512,512,8192 2,512,512,4096 2,512,512,2048 2>&1 | tail -3
  HB_WGRAD_BN=$1 HB_MAX_SPLITS=$2 timeout -s KILL 60 python scripts/gemm_phases.py 2,512,512,8192 2>&1 | tail -9
done
