#!/bin/bash
mkdir -p gpurun_out
timeout -s KILL 700 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/gpu_tests.log 2>&1; tail -1 gpurun_out/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 300 gpurun_out/bench_default.err
timeout -s KILL 300 python bench.py --policy minibatch --steps 10 --warmup 3 --ttt-epochs 0 > gpurun_out/bench_mb_covtype.json 2> gpurun_out/bench_mb_covtype.err
timeout -s KILL 600 python bench.py --config realsim --policy minibatch --steps 5 --warmup 3 --ttt-epochs 0 > gpurun_out/bench_mb_realsim.json 2> gpurun_out/bench_mb_realsim.err
