#!/bin/bash
# scratch driver for one gpurun call (edited per experiment); default: build + smoke, the GPU suite, the bench lines
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > $O/full.log
for c in c5 c2 c3; do timeout 900 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
