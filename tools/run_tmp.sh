#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > $O/full.log
timeout 900 python bench.py > $O/bench_c5.json 2> $O/bench_c5.err
timeout 900 python bench.py --config c2 > $O/bench_c2.json 2> $O/bench_c2.err
