#!/bin/bash
O=gpurun_out
timeout 900 python bench.py --config c4 --steps 5 > $O/b_c4.json 2> $O/b_c4.err
timeout 600 python bench.py --steps 5 --no-cpu-baseline > $O/b_c5y.json 2> $O/b_c5y.err
