#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
python -m pytest tests -m gpu -q 2>&1 | grep -v "^$" | tail -30 > $O/t10.log
python bench.py --config c3 --steps 5 --warmup 3 --no-cpu-baseline > $O/b_c3e.json 2> $O/b_c3e.err
