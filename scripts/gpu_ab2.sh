#!/bin/bash
echo "== main"; timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 2048,8192 2>&1 | grep -A12 "^---\|graph"
echo "== fakesig"; HB_LIB=$PWD/paper_conf_ipps_marws21_b200/variants/libhogbatch_fakesig.so timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 8192 2>&1 | grep -A12 "^---\|graph"
timeout -s KILL 300 python -m pytest tests/test_gpu_rowchain.py tests/test_gpu_step.py -q -x 2>&1 | tail -2
