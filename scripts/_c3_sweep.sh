export HB_LIB=paper_conf_ipps_marws21_b200/variants/libhogbatch_tuning.so
for cfg in "X=1" "HB_FWD_BN=256" "HB_FWD_BN=64" "HB_WGRAD_BN=128" "HB_WGRAD_BN=64" "HB_MAX_SPLITS=1" "HB_FWD_BN=256 HB_WGRAD_BN=128"; do
  echo "== $cfg"; env $cfg timeout 300 python bench.py --config w8a --policy minibatch --steps 20 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print(round(d['value']/1e6,2),'M/s', round(d['tc_peak_frac'],3), 'ms/step', round(d['ms_per_step'],3)); print({k:(v['ms_per_step'],v['TFLOP/s']) for k,v in list(r['classes'].items())[:8]})"
done
