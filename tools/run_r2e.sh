#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build.log 2>&1
python -m pytest tests/test_gpu_select.py tests/test_gpu_fullsize.py::test_full_size_selection tests/test_gpu_decisions.py::test_topk_decisions_k_sweep "tests/test_gpu_dp.py::test_sharded_selection_k12_equals_single_gpu" tests/test_gpu_stem.py -q -x 2>&1 | grep -v "^$" | tail -20 > $O/t9.log
bash tools/ncu_one.sh self2 'select_fused|topk|radix|emit|project_ref|ref_norm|transpose_w' 0 16 -- python bench.py --config c5 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep --no-graph --profile-steps 1
