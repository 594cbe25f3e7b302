#!/bin/bash
# Round-trip validation of HEAD: all GPU tests, default bench line, mini-batch bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout -s KILL 700 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/gpu_tests.log 2>&1
tail -5 gpurun_out/gpu_tests.log
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
tail -c 800 gpurun_out/bench_default.json; tail -3 gpurun_out/bench_default.err
timeout -s KILL 300 python bench.py --policy minibatch --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_mb.json 2> gpurun_out/bench_mb.err
tail -c 400 gpurun_out/bench_mb.json
