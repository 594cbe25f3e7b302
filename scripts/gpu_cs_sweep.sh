#!/bin/bash
# fused chain: cluster size sweep per batch size (graph device time)
for cs in 2 4 8; do
  echo "== HB_RC_CS=$cs"; HB_RC_CS=$cs timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 32,256,1024,2048,4096,8192 2>&1 | grep graph
done
echo "== auto"; timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 32,256,1024,2048,4096,8192 2>&1 | grep graph
echo "== unfused"; HB_ROWCHAIN=0 timeout -s KILL 100 python scripts/rc_probe.py 54,512,512,512,512,7 32,256,1024,2048,4096,8192 2>&1 | grep graph
timeout -s KILL 240 python -m pytest tests/test_gpu_rowchain.py -x -q --timeout 120 2>&1 | tail -3
