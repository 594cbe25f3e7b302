#!/bin/bash
# One GPU round trip: parity tests, benches, ncu launch list (cold, serialised).
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
timeout -s KILL 300 python bench.py --policy minibatch --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_mb.json 2> gpurun_out/bench_mb.err
tail -c 1500 gpurun_out/bench_mb.json
timeout -s KILL 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ad.json 2> gpurun_out/bench_ad.err
tail -c 600 gpurun_out/bench_ad.json
timeout -s KILL 400 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_mb.csv python bench.py --policy minibatch --steps 1 --warmup 0 --e2e-steps 0 --no-prof --no-cpu-baseline > /dev/null 2>&1
echo ncu rc=$?
