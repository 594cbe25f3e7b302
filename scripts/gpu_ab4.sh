#!/bin/bash
bash scripts/gpu_dw_ph2.sh 2>&1 | grep -A9 "=="
for k in 0 2; do echo "== KORDER=$k"; HB_RC_KORDER=$k timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 2048,8192 2>&1 | grep -A10 "^---\|graph"; done
timeout -s KILL 400 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -2
