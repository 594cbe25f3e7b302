#!/bin/bash
# A/B of the pair-tile raster group (default 8 pair rows vs the g16pair variant): C4 bench lines
# (alternating, two reps) and ncu DRAM bytes of the layer-1 forward / dW launches of one C4 step
mkdir -p gpurun_out/abg; O=gpurun_out/abg
V=paper_conf_ipps_marws21_b200/variants/libhogbatch_g16pair.so
for rep in 1 2; do for lib in "" "$V"; do
  HB_LIB=$lib timeout 600 python bench.py --steps 8 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --no-prof --e2e-steps 0 > $O/b.json 2>$O/b.err
  python - "${lib:-default}" <<'PY'
import json, sys
d = json.loads(open("gpurun_out/abg/b.json").read().strip().splitlines()[-1])
print(sys.argv[1].split("/")[-1], "value", round(d["value"] / 1e6, 4), "M  ms", round(d["ms_per_step"], 3), "clk", d["clocks"]["sm_mhz"])
PY
done; done
for lib in "" "$V"; do
  HB_LIB=$lib timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:tc_gemm_kernel -c 14 --csv python scripts/c4_step.py 1 2>/dev/null | grep -E "tc_gemm" | \
    python -c "
import sys, csv
rows = list(csv.reader(sys.stdin))
v = {}
for r in rows:
    k = (r[0], r[4][:60])
    v.setdefault(k, {})[r[-3]] = r[-1]
for k, m in v.items(): print('${lib:-default}'.split('/')[-1], k[0], k[1], m)
" | head -30
done
