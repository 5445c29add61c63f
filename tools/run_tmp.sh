#!/bin/bash
O=gpurun_out
export N=1024 SHAPES=0 MODES=1 REPS=20
ADAINF_WSKX=1 timeout 900 python -m pytest tests/test_gpu_conv.py -q -x -k "window" 2>&1 | tail -3 > $O/conv.log
for r in 1 2; do
for kx in 0 1; do
ADAINF_WSKX=$kx timeout 300 python tools/time_layers.py 2>&1 | sed "s/^/kx=$kx /"
done
done > $O/tl.log
