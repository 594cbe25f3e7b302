#!/bin/bash
# parity (all GPU tests) + fused/unfused step probe
timeout -s KILL 400 python -m pytest tests -m gpu -q -x --timeout 200 2>&1 | tail -3
for rc in 1 0; do echo "== HB_ROWCHAIN=$rc"; HB_ROWCHAIN=$rc timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 32,256,2048,4096,8192 2>&1 | grep graph; done
