#!/bin/bash
# A/B: 8 vs 16 epilogue warps in the tcgen05 GEMM (variant library via HB_LIB): GPU tests on the
# variant, then bench lines of both builds
mkdir -p gpurun_out/ab; O=gpurun_out/ab
V=${VARIANT:-paper_conf_ipps_marws21_b200/variants/libhogbatch_epi16.so}
[ -z "$NO_TESTS" ] && HB_LIB=$V timeout -s KILL 1200 python -m pytest tests -m gpu -q -x --timeout 600 > $O/tests_epi16.log 2>&1; tail -2 $O/tests_epi16.log
line() { python - "$1" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/ab/b.json").read().strip().splitlines()[-1])
print(sys.argv[1], "value", round(d["value"] / 1e6, 3), "M  ms", round(d["ms_per_step"], 3), "tc", round(d.get("tc_peak_frac") or 0, 4))
PY
}
for c in "--config w8a --policy minibatch" "--config covtype --policy minibatch" "--config covtype" ""; do
  for lib in "" "$V"; do
    HB_LIB=$lib timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof --e2e-steps 0 $c > $O/b.json 2>$O/b.err
    line "[$c] lib=${lib:-default}"
  done
done
for lib in "" "$V"; do HB_LIB=$lib STEPS=200 timeout 300 python scripts/small_batch_probe.py 32,256,2048 2>&1 | tail -3 | tr '\n' ' '; echo " lib=${lib:-default}"; done
