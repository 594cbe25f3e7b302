#!/bin/bash
for cfg in "256 4" "128 4" "64 4"; do
  set -- $cfg
  echo "== HB_WGRAD_BN=$1 HB_MAX_SPLITS=$2"
  HB_WGRAD_BN=$1 HB_MAX_SPLITS=$2 timeout -s KILL 60 python scripts/gemm_bench.py 2,512,512,8192 2>&1 | tail -1
  HB_WGRAD_BN=$1 HB_MAX_SPLITS=$2 timeout -s KILL 60 python scripts/gemm_phases.py 2,512,512,8192 2>&1 | tail -9
done
