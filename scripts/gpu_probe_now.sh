#!/bin/bash
mkdir -p gpurun_out
timeout -s KILL 120 python scripts/rc_probe.py 54,512,512,512,512,7 256,2048,8192 > gpurun_out/rc_probe.log 2>&1
tail -40 gpurun_out/rc_probe.log
