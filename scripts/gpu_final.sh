#!/bin/bash
# Round-end measurement pass (one gpurun call): smoke, GPU tests, bench lines of every config,
# reference arm, ncu launch list of the default bench command, ncu --set full of a C4 step.
mkdir -p gpurun_out/final
rm -rf gpurun_out/quick
O=gpurun_out/final
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout -s KILL 1500 python -m pytest tests -m gpu -q -rA --timeout 600 -s > $O/gpu_tests.log 2>&1
grep -E "max rel|normwise|beta|passed|failed" $O/gpu_tests.log | tail -12
run() { name=$1; shift; timeout -s KILL 900 python bench.py "$@" > $O/bench_$name.json 2> $O/bench_$name.err; echo "bench $name rc=$?"; }
run c4_default
run c2_adaptive --config covtype
run c2_minibatch --config covtype --policy minibatch --ttt-epochs 0
run c3_minibatch --config w8a --policy minibatch --ttt-epochs 0
run c3_adaptive --config w8a
run c1_tiny --config tiny --ttt-epochs 0
timeout -s KILL 600 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference rc=$?"
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c4.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --ttt-epochs 0 --e2e-steps 0 --no-prof > $O/ncu_bench.log 2>&1; echo "launch list rc=$?"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:"tc_gemm_kernel|head_" -c 14 -f -o $O/c4_step \
  python scripts/c4_step.py 1 > $O/ncu_c4.log 2>&1; echo "ncu full rc=$?"
# summarise on the box (gpurun copies back <= 64 MiB): per-launch summary, raw metrics, details page of
# the longest launch; the .ncu-rep itself stays behind
python scripts/ncu_traffic.py $O/c4_step.ncu-rep realsim > $O/ncu_c4_summary.txt 2>&1; cp profiles/ncu_traffic.json $O/ 2>/dev/null
ncu -i $O/c4_step.ncu-rep --page raw --csv > $O/ncu_c4_raw.csv 2>/dev/null
ncu -i $O/c4_step.ncu-rep --page details --print-details all -k regex:tc_gemm_kernel --launch-skip 0 --launch-count 1 > $O/ncu_c4_l1fwd_details.txt 2>/dev/null
ncu -i $O/c4_step.ncu-rep --page details > $O/ncu_c4_details.txt 2>/dev/null
rm -f $O/c4_step.ncu-rep
timeout -s KILL 300 python scripts/softmax_probe.py > $O/softmax.json 2>&1; tail -1 $O/softmax.json
STEPS=200 timeout -s KILL 300 python scripts/small_batch_probe.py 32,256,1024,2048,4096,8192 > $O/small_batch.jsonl 2>&1; tail -2 $O/small_batch.jsonl
