#!/bin/bash
echo "== parts 4 (main)"; timeout -s KILL 60 python scripts/rc_probe.py 54,512,512,512,512,7 4096,8192 2>&1 | grep -A10 "^---\|graph"
echo "== parts 2"; HB_LIB=$PWD/paper_conf_ipps_marws21_b200/variants/libhogbatch_parts2.so timeout -s KILL 60 python scripts/rc_probe.py 54,512,512,512,512,7 4096,8192 2>&1 | grep graph
timeout -s KILL 300 python -m pytest tests/test_gpu_rowchain.py -q -x --timeout 200 2>&1 | tail -1
