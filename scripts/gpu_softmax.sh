python -m pytest tests/test_gpu_step.py -q -x -k "delicious or many_classes" 2>&1 | tail -3
python scripts/softmax_probe.py
ncu --set full --clock-control none -k regex:softmax_xent -c 1 -f -o gpurun_out/softmax983 python scripts/softmax_probe.py > gpurun_out/ncu_softmax.log 2>&1; echo ncu rc=$?
