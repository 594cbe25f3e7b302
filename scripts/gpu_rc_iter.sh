#!/bin/bash
# rowchain iteration: fused parity tests (hang-guarded), then the probe
mkdir -p gpurun_out
timeout -s KILL 240 python -m pytest tests/test_gpu_rowchain.py -x -q --timeout 120 > gpurun_out/rc_tests.log 2>&1
echo "rowchain tests rc=$?"; tail -15 gpurun_out/rc_tests.log
HB_ROWCHAIN=1 timeout -s KILL 120 python scripts/rc_probe.py ${PROBE_DIMS:-54,512,512,512,512,7} > gpurun_out/probe_rc1.txt 2>&1
cat gpurun_out/probe_rc1.txt
