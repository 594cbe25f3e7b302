#!/bin/bash
# rowchain bring-up: fused-path parity tests (hang-guarded), then the step/hogbatch suites
mkdir -p gpurun_out
timeout -s KILL 240 python -m pytest tests/test_gpu_rowchain.py -x -q --timeout 120 > gpurun_out/rc_tests.log 2>&1
echo "rowchain tests rc=$?"; tail -25 gpurun_out/rc_tests.log
timeout -s KILL 400 python -m pytest tests -m gpu -q --timeout 200 > gpurun_out/gpu_tests.log 2>&1
echo "gpu tests rc=$?"; tail -15 gpurun_out/gpu_tests.log
