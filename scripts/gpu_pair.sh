#!/bin/bash
# A/B of the CTA-pair dW GEMMs in the fused step (HB_DW_PAIR) + fused-path parity with pairs
for p in 1 0 1; do HB_DW_PAIR=$p timeout -s KILL 60 python scripts/rc_probe.py 54,512,512,512,512,7 4096,8192 2>&1 | grep graph | sed "s/^/pair$p /"; done
HB_DW_PAIR=1 timeout -s KILL 300 python -m pytest tests/test_gpu_rowchain.py tests/test_gpu_hogbatch.py -q -x --timeout 200 2>&1 | tail -3
