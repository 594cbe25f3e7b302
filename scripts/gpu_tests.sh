#!/bin/bash
# GPU test pass: smoke + the whole -m gpu suite (verbose, with the parity tests' printed errors).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout -s KILL 1500 python -m pytest tests -m gpu -q -rA --timeout 600 -s ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/gpu_tests.log 2>&1
grep -E "max rel|normwise|passed|failed|Error|assert" gpurun_out/gpu_tests.log | tail -40
