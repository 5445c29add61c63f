#!/bin/bash
# Round-2 profiling evidence (run under gpurun from the repo root): bench lines (c5 default, c2, c3), the ncu launch
# list of the bench command (gpu__time_duration only, cold + serialised: compare shares), per-launch DRAM traffic of a
# C5-shaped step, and ncu --set full captures (raw + SASS) of the top kernels.
# usage: tools/profile_r2.sh TAG
set -u
TAG=${1:-r2a}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1
for c in c5 c2 c3; do
  timeout 900 python bench.py --config $c > $O/${TAG}_bench_$c.json 2> $O/${TAG}_bench_$c.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv \
  --log-file $O/${TAG}_bench_launch_list.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-sweep \
  > $O/${TAG}_bench_under_ncu.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 \
  --csv --log-file $O/${TAG}_c3_launch_list.csv python bench.py --config c3 --steps 1 --warmup 3 --no-e2e \
  --no-cpu-baseline --no-sweep > $O/${TAG}_c3_under_ncu.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed
timeout 900 ncu --metrics $M --clock-control none --nvtx --nvtx-include "profiled/" --csv \
  --log-file $O/${TAG}_step_traffic.csv python tools/profile_step.py --steps 2 --k 8192 --taus 0.24,0.40,0.61 \
  > $O/${TAG}_step.log 2>&1
for K in stem_fwd_kernel conv_ws_tma_kernel conv_umma_kernel conv_wgrad_tma_kernel conv_wgrad_win_tma_kernel conv_dualm_kernel exit_fused_kernel; do
  bash tools/ncu_one.sh ${TAG}_$K "$K" 2 1 -- python tools/profile_step.py --steps 2 --k 1024
done
bash tools/ncu_one.sh ${TAG}_stem_wgrad_kernel stem_wgrad_kernel 0 1 -- python tools/profile_step.py --steps 1 --k 1024 --train-only
bash tools/ncu_one.sh ${TAG}_sgd_kernel sgd_kernel 0 1 -- python tools/profile_step.py --steps 1 --k 1024 --train-only
bash tools/ncu_one.sh ${TAG}_conv3_pool_kernel conv3_pool_kernel 0 3 -- python tools/time_conv3pool.py
bash tools/ncu_one.sh ${TAG}_select_fused_kernel select_fused_kernel 0 1 -- python tools/time_select.py
echo done
