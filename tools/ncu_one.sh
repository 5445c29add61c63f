#!/bin/bash
# ncu --set full of a few launches of one kernel, exported to CSV on the box (raw + SASS source with stalls).
# usage: tools/ncu_one.sh TAG KERNEL_REGEX SKIP COUNT -- cmd...
TAG=$1; KRE=$2; SKIP=$3; CNT=$4; shift 5
O=gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$KRE" -s $SKIP -c $CNT -o $O/$TAG -f "$@" > $O/$TAG.log 2>&1
ncu -i $O/$TAG.ncu-rep --page raw --csv > $O/${TAG}_raw.csv 2>/dev/null
for i in $(seq 0 $((CNT-1))); do
  ncu -i $O/$TAG.ncu-rep --page source --csv --print-source sass --launch-skip $i --launch-count 1 > $O/${TAG}_sass$i.csv 2>/dev/null
done
rm -f $O/$TAG.ncu-rep
