#!/bin/bash
HB_WGRAD_BN=256 HB_MAX_SPLITS=4 timeout -s KILL 60 python scripts/gemm_phases.py 2,512,512,8192 2>&1 | tail -13
for k in 0 2; do echo "== KORDER=$k"; HB_RC_KORDER=$k timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 8192 2>&1 | grep -A10 "^---\|graph"; done
timeout -s KILL 400 python -m pytest tests/test_gpu_rowchain.py -q -x --timeout 300 2>&1 | tail -2
