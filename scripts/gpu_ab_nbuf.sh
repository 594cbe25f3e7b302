#!/bin/bash
# A/B: CTA-pair tile epilogue staging (1 buffer vs double-buffered H; + staged sigma'): hidden-layer
# phase timeline (tuning builds) and C4 bench lines (alternating)
mkdir -p gpurun_out/abn; O=gpurun_out/abn
V=paper_conf_ipps_marws21_b200/variants
for t in tuning tuning_nbuf2; do
  echo "== $t"; HB_GEMM_PAIR=1 HB_LIB=$V/libhogbatch_$t.so timeout 120 python scripts/gemm_phases.py 0,8192,4096,4096 1,8192,4096,4096 2>&1 | grep -E "span|mma_issued|epi_done_t[0-2]"
done
for rep in 1 2; do for lib in "" "$V/libhogbatch_nbuf2.so" "$V/libhogbatch_nbuf2out2.so"; do
  HB_LIB=$lib timeout 600 python bench.py --steps 8 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof --e2e-steps 0 > $O/b.json 2>$O/b.err
  python - "${lib:-default}" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/abn/b.json").read().strip().splitlines()[-1])
print(sys.argv[1].split("/")[-1], "value", round(d["value"] / 1e6, 4), "M  ms", round(d["ms_per_step"], 3), "clk", d["clocks"]["sm_mhz"])
PY
done; done
