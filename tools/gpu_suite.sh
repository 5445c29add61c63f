#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q --durations=15 2>&1 | grep -v "^$" | tail -60 > $O/full.log
