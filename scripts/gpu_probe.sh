mkdir -p gpurun_out
HB_ROWCHAIN=1 timeout -s KILL 120 python scripts/rc_probe.py > gpurun_out/probe_rc1.txt 2>&1
HB_ROWCHAIN=0 timeout -s KILL 120 python scripts/rc_probe.py > gpurun_out/probe_rc0.txt 2>&1
cat gpurun_out/probe_rc1.txt gpurun_out/probe_rc0.txt
