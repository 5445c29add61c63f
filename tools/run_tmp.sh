#!/bin/bash
O=gpurun_out
export N=1024 SHAPES=1 MODES=1 REPS=20
for x in 0 4 8 12; do
ADAINF_EXP=$x timeout 300 python tools/time_layers.py 2>&1 | grep dgrad | sed "s/^/exp=$x /"
done > $O/spexp.log
