#!/bin/bash
# Round-end artefacts: GPU tests, bench lines for every config, sweep, launch list, ncu captures.
mkdir -p gpurun_out
timeout -s KILL 700 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/gpu_tests.log 2>&1; tail -1 gpurun_out/gpu_tests.log
timeout -s KILL 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 200 gpurun_out/bench_default.err
timeout -s KILL 300 python bench.py --policy minibatch --steps 10 --warmup 3 --ttt-epochs 0 > gpurun_out/bench_mb_covtype.json 2> gpurun_out/bench_mb_covtype.err
timeout -s KILL 300 python bench.py --config w8a --steps 10 --warmup 3 --ttt-epochs 20 > gpurun_out/bench_ad_w8a.json 2> gpurun_out/bench_ad_w8a.err; tail -c 200 gpurun_out/bench_ad_w8a.err
timeout -s KILL 300 python bench.py --config w8a --policy minibatch --steps 10 --warmup 3 --ttt-epochs 0 > gpurun_out/bench_mb_w8a.json 2> gpurun_out/bench_mb_w8a.err
timeout -s KILL 300 python bench.py --config tiny --steps 10 --warmup 3 --ttt-epochs 0 > gpurun_out/bench_tiny.json 2> gpurun_out/bench_tiny.err; tail -c 200 gpurun_out/bench_tiny.err
timeout -s KILL 600 python bench.py --config realsim --policy minibatch --steps 5 --warmup 3 --ttt-epochs 0 > gpurun_out/bench_mb_realsim.json 2> gpurun_out/bench_mb_realsim.err; tail -c 200 gpurun_out/bench_mb_realsim.err
timeout -s KILL 600 python scripts/sweep.py 32,256,2048,8192,65536 256,512,1024,4096,8192 > gpurun_out/sweep.jsonl 2> gpurun_out/sweep.err; tail -c 200 gpurun_out/sweep.err
timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 4096,8192 > gpurun_out/rc_probe.log 2>&1; grep graph gpurun_out/rc_probe.log
timeout -s KILL 400 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_minibatch.csv \
  python bench.py --policy minibatch --steps 1 --warmup 0 --e2e-steps 0 --no-prof --no-cpu-baseline --ttt-epochs 0 > /dev/null 2>&1; echo "ncu launches rc=$?"
timeout -s KILL 400 ncu --set full --import-source on --clock-control none -k regex:"rowchain|tc_gemm" -s 12 -c 6 \
  -o gpurun_out/step_full_8192 -f python scripts/rc_one.py 8192 > gpurun_out/ncu_step.log 2>&1; echo "ncu full rc=$?"
