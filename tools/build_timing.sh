#!/bin/bash
# Build an instrumented copy of libadainf.so (ADAINF_TIMING) into /tmp/adainf_timing/ for role-wait analysis.
set -e
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OUT=${1:-$ROOT/tools/timing_build}
mkdir -p "$OUT"
NCCL=$(python -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])")
objs=""
for f in "$ROOT"/paper_conf_sigcomm_shubhas23_b200/csrc/*.cu; do
  o="$OUT/$(basename "$f" .cu).o"
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -DADAINF_TIMING -rdc=false \
    -I "$ROOT/paper_conf_sigcomm_shubhas23_b200/csrc" -I "$ROOT/include" -I "$NCCL/include" -DADAINF_WITH_NCCL=1 -c "$f" -o "$o" &
  objs="$objs $o"
done
wait
nvcc -shared -gencode arch=compute_100a,code=sm_100a -o "$OUT/libadainf.so" $objs -lcudart -L "$NCCL/lib" -l:libnccl.so.2 -Xlinker -rpath="$NCCL/lib"
echo "$OUT/libadainf.so"
