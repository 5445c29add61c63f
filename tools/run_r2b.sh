#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
python -m pytest tests/test_gpu_select.py tests/test_gpu_fullsize.py::test_full_size_selection tests/test_gpu_decisions.py tests/test_gpu_variants.py tests/test_gpu_dp.py tests/test_gpu_sched.py -q -s 2>&1 | grep -v "^$" | tail -60 > $O/t6.log
python bench.py --config c5 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/b_c5b.json 2> $O/b_c5b.err
