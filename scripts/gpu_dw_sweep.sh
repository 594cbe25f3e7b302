#!/bin/bash
# dW tile / split sweep for the fused path's concurrent dW GEMMs (C2 shape)
for cfg in "0 0" "64 4" "128 4" "256 4" "256 2" "256 8" "128 8" "128 2"; do
  set -- $cfg
  echo "== HB_RC_WGRAD_BN=$1 HB_RC_WGRAD_S=$2"
  HB_RC_WGRAD_BN=$1 HB_RC_WGRAD_S=$2 timeout -s KILL 120 python scripts/rc_probe.py 54,512,512,512,512,7 32,256,2048,8192 2>&1 | grep graph
done
echo "== unfused"
HB_ROWCHAIN=0 timeout -s KILL 120 python scripts/rc_probe.py 54,512,512,512,512,7 32,256,2048,8192 2>&1 | grep graph
