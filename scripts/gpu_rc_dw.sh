#!/bin/bash
# tuning build: C2 fused-step dW GEMM tile width x splits (HB_RC_WGRAD_BN / HB_RC_WGRAD_S)
export HB_LIB=paper_conf_ipps_marws21_b200/variants/libhogbatch_tuning.so
mkdir -p gpurun_out/rcdw; O=gpurun_out/rcdw/sweep.txt; : > $O
timeout 120 python scripts/rc_dw_sweep.py >> $O 2>&1
for bn in 128 256; do for s in 2 4 8; do
  HB_RC_WGRAD_BN=$bn HB_RC_WGRAD_S=$s timeout 120 python scripts/rc_dw_sweep.py >> $O 2>&1
done; done
HB_DW_PAIR=1 timeout 120 python scripts/rc_dw_sweep.py >> $O 2>&1
cat $O
