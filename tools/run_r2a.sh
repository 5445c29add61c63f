#!/bin/bash
# round-2 GPU batch A: c3 bench, new parity tests, stem ncu captures
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1
python bench.py --config c3 --steps 5 --warmup 3 --no-cpu-baseline > $O/b_c3.json 2> $O/b_c3.err
python -m pytest tests/test_gpu_variants.py tests/test_gpu_decisions.py tests/test_gpu_model.py -q -s 2>&1 | tail -40 > $O/t3.log
bash tools/ncu_one.sh stemf 'stem_fwd' 1 1 -- python tools/profile_step.py --train-only --steps 2 --k 1024
bash tools/ncu_one.sh stemw 'stem_wgrad' 1 1 -- python tools/profile_step.py --train-only --steps 2 --k 1024
