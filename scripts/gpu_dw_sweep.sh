#!/bin/bash
# dW / forward GEMM tile-choice sweep (tuning build): C3 hidden shapes and the C4 hidden dW
export HB_LIB=paper_conf_ipps_marws21_b200/variants/libhogbatch_tuning.so
mkdir -p gpurun_out/sweep; O=gpurun_out/sweep/dw.txt; : > $O
for bn in 64 128 256; do for s in 1 2 4 8; do for dp in 0 1; do
  echo "C3 dW bn=$bn S=$s dwpair=$dp: $(HB_WGRAD_BN=$bn HB_FORCE_SPLITS=$s HB_DW_PAIR=$dp timeout 60 python scripts/gemm_bench.py 2,1024,1024,8192 2>&1 | tail -1)" >> $O
done; done; done
for bn in 128 256; do for s in 1 2; do for gp in 0 1; do
  echo "C4 hidden dW bn=$bn S=$s gemmpair=$gp: $(HB_WGRAD_BN=$bn HB_FORCE_SPLITS=$s HB_GEMM_PAIR=$gp timeout 60 python scripts/gemm_bench.py 2,4096,4096,8192 2>&1 | tail -1)" >> $O
done; done; done
for bn in 64 128 256; do for gp in 0 1; do
  echo "C3 fwd bn=$bn gemmpair=$gp: $(HB_FWD_BN=$bn HB_GEMM_PAIR=$gp timeout 60 python scripts/gemm_bench.py 0,8192,1024,1024 1,8192,1024,1024 2>&1 | tail -2 | tr '\n' ' ')" >> $O
done; done
cat $O
