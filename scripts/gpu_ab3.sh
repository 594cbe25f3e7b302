#!/bin/bash
echo "== main"; timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 8192 2>&1 | grep -A16 "cta0\|graph"
echo "== no S store"; HB_LIB=$PWD/paper_conf_ipps_marws21_b200/variants/libhogbatch_nos.so timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 8192 2>&1 | grep -A12 "^---\|graph"
