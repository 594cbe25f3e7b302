#!/bin/bash
for v in 1 0; do echo "== HB_RC_S_TMA=$v"; HB_RC_S_TMA=$v timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 8192 2>&1 | grep -A10 "^---\|graph"; done
timeout -s KILL 400 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -2
