timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for bn in 256 128; do echo "== FWD_BN $bn"; HB_FWD_BN=$bn HB_LIB=paper_conf_ipps_marws21_b200/variants/libhogbatch_tuning.so python scripts/gemm_phases.py 0,8192,1024,1024 1,8192,1024,1024 | grep -E "span|mma_issued_t[0-1]|epi_done_t[0-1]"; done
for env in "X=1" "HB_FWD_BN=256"; do for cfg in "--config w8a --policy minibatch" "--config realsim"; do
  echo "== $env $cfg"; env $env HB_LIB=paper_conf_ipps_marws21_b200/variants/libhogbatch_tuning.so timeout 300 python bench.py $cfg --steps 10 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print(round(d['value']/1e6,3),'M/s', round(d['tc_peak_frac'],3), 'ms/step', round(d['ms_per_step'],3), 'clk', d['clocks']['sm_mhz']); print({k:(v['ms_per_step'],v['TFLOP/s']) for k,v in list(r['classes'].items())[:7]})"
done; done
