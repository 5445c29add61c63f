#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
python -m pytest tests/test_gpu_stem.py tests/test_gpu_model.py tests/test_gpu_decisions.py::test_exit_decisions_tau_sweep tests/test_gpu_select.py -q -x 2>&1 | grep -v "^$" | tail -30 > $O/t8.log
python bench.py --config c5 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > $O/b_c5d.json 2> $O/b_c5d.err
ADAINF_STEM_V2=0 python bench.py --config c5 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > $O/b_c5d_v1.json 2> $O/b_c5d_v1.err
bash tools/ncu_one.sh self 'select_fused|topk|radix|emit|project_ref' 0 8 -- python bench.py --config c5 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep --no-graph --profile-steps 1
