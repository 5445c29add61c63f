#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
python -m pytest tests/test_gpu_model.py tests/test_gpu_select.py tests/test_gpu_fullsize.py tests/test_gpu_decisions.py tests/test_gpu_dag.py tests/test_gpu_graph.py tests/test_gpu_sched.py -q -x 2>&1 | grep -v "^$" | tail -30 > $O/t7.log
python bench.py --config c2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/b_c2c.json 2> $O/b_c2c.err
ADAINF_EXIT_FUSED=0 python bench.py --config c2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/b_c2c_nofuse.json 2> $O/b_c2c_nofuse.err
python bench.py --config c5 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/b_c5c.json 2> $O/b_c5c.err
