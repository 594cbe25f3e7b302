#!/bin/bash
for k in 0 1; do echo "== HB_RC_KORDER=$k"; HB_RC_KORDER=$k timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 256,2048,8192 2>&1 | grep -A12 "^---\|graph"; done
HB_RC_KORDER=1 timeout -s KILL 300 python -m pytest tests/test_gpu_rowchain.py -q -x 2>&1 | tail -2
bash scripts/gpu_dw_sweep.sh
