#!/bin/bash
HB_WGRAD_BN=256 HB_MAX_SPLITS=4 timeout -s KILL 60 python scripts/gemm_phases.py 2,512,512,8192 2>&1 | tail -13
timeout -s KILL 60 python scripts/rc_probe.py 54,512,512,512,512,7 4096,8192 2>&1 | grep graph
timeout -s KILL 400 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -2
