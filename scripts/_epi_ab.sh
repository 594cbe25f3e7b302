for lib in "" "paper_conf_ipps_marws21_b200/variants/libhogbatch_noTMA128.so" "paper_conf_ipps_marws21_b200/variants/libhogbatch_ring220.so"; do
 for cfg in "--config w8a --policy minibatch" "--config covtype --policy minibatch" "--config realsim"; do
  echo "== lib=${lib:-default} $cfg"; HB_LIB=$lib timeout 300 python bench.py $cfg --steps 10 --warmup 3 --no-cpu-baseline --ttt-epochs 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print(round(d['value']/1e6,3),'M/s', round(d['tc_peak_frac'],3), 'ms/step', round(d['ms_per_step'],3), 'clk', d['clocks']['sm_mhz']); print({k:(v['ms_per_step'],v['TFLOP/s']) for k,v in list(r['classes'].items())[:6]})"
 done
done
