#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
./tools/exp_stem_mma > $O/exp_stem_mma.log 2>&1
python tools/time_det_layers.py > $O/det_layers.log 2>&1
