#!/bin/bash
# Round measurement pass: GPU tests, default bench line (C4), the ncu launch list of the bench
# command, and one `ncu --set full` capture of a C4 step's 14 GEMM launches.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
if [ -z "$SKIP_TESTS" ]; then
timeout -s KILL 1500 python -m pytest tests -m gpu -q -rA --timeout 600 -s > gpurun_out/gpu_tests.log 2>&1
grep -E "max rel|normwise|beta|passed|failed|Error" gpurun_out/gpu_tests.log | tail -20
fi
timeout -s KILL 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -c 1500 gpurun_out/bench.json; tail -3 gpurun_out/bench.err
if [ -z "$SKIP_NCU" ]; then
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --ttt-epochs 0 --e2e-steps 0 --no-prof ${BENCH_ARGS} > gpurun_out/ncu_bench.log 2>&1
echo "launches rc=$?"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:tc_gemm_kernel -c 14 -f -o gpurun_out/c4_step \
  python scripts/c4_step.py 1 > gpurun_out/ncu_c4.log 2>&1
echo "ncu full rc=$?"
fi
