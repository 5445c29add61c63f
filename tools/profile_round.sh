#!/bin/bash
# One GPU call's worth of profiling evidence for profiles/ (run under gpurun from the repo root).
#   1. launch list of one bench-shaped step (infer 256 + retrain 1024) with time, DRAM bytes, tensor-pipe %
#      (cold-cache, serialised: compare shares, not absolutes)
#   2. launch list of the bench command itself (gpu__time_duration only, as the recipe asks)
#   3. ncu --set full of the top conv kernel(s) (a few launches)
# usage: tools/profile_round.sh TAG [kernel-regex]
set -u
TAG=${1:-r1}
KRE=${2:-regex:conv_}
O=gpurun_out
mkdir -p $O
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed
timeout 600 ncu --metrics $M --clock-control none --nvtx --nvtx-include "profiled/" --csv \
  --log-file $O/${TAG}_step_traffic.csv python tools/profile_step.py --steps 3 > $O/${TAG}_step.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
  --log-file $O/${TAG}_bench_launch_list.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline \
  > $O/${TAG}_bench_under_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "profiled/" -k "$KRE" -c ${NFULL:-6} \
  -o $O/${TAG}_full -f python tools/profile_step.py --train-only --steps 2 > $O/${TAG}_full.log 2>&1

# keep the bring-back small: export the full capture's raw metrics (+ per-kernel SASS stall tops) as CSV and
# drop the report unless it is small
ncu -i $O/${TAG}_full.ncu-rep --page raw --csv > $O/${TAG}_full_raw.csv 2>/dev/null
sz=$(stat -c %s $O/${TAG}_full.ncu-rep 2>/dev/null || echo 0)
if [ "$sz" -gt 30000000 ]; then rm -f $O/${TAG}_full.ncu-rep; fi
echo done
