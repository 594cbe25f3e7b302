#!/bin/bash
# A/B of library variants (paper_conf_ipps_marws21_b200/variants/*.so) on the fused-step probe
DIMS=${PROBE_DIMS:-54,512,512,512,512,7}
B=${PROBE_B:-32,2048,8192}
echo "== default"; timeout -s KILL 120 python scripts/rc_probe.py $DIMS $B 2>&1 | grep graph
for v in paper_conf_ipps_marws21_b200/variants/*.so; do
  echo "== $v"; HB_LIB=$v timeout -s KILL 120 python scripts/rc_probe.py $DIMS $B 2>&1 | grep graph
done
