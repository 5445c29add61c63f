#!/bin/bash
O=gpurun_out
timeout 600 python -m pytest tests/test_gpu_conv.py -q -x -k "dgrad" 2>&1 | tail -2 > $O/sp_tests.log
export N=1024 SHAPES=1,4,7 MODES=1 REPS=20
for r in 1 2; do
ADAINF_LIB=/root/repo/_variants/base/libadainf.so timeout 300 python tools/time_layers.py 2>&1 | grep dgrad | sed "s/^/base /"
timeout 300 python tools/time_layers.py 2>&1 | grep dgrad | sed "s/^/new  /"
done > $O/sp_time.log
