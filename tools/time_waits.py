"""Barrier-wait attribution of the layer-1 window kernel (conv_ws_tma_kernel) from a -DADAINF_TIMING build:
  ADAINF_BUILD_OUT=/tmp/tv/libadainf.so ADAINF_BUILD_FLAGS=-DADAINF_TIMING python -m paper_conf_sigcomm_shubhas23_b200.build
  ADAINF_LIB=/tmp/tv/libadainf.so python tools/time_waits.py
Slots (cycles summed over warps / CTAs, printed per tile and per CTA): 0 producer wempty, 1 MMA tempty,
2 MMA wfull, 3 epilogue tfull, 4 epilogue efull, 5 epilogue pre-store barrier, 6 epilogue store barrier,
7 MMA-warp loop total."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
if os.environ.get("ADAINF_LIB"):
    B.LIB_PATH = os.environ["ADAINF_LIB"]

n = int(os.environ.get("N", "1024"))
H, Cc = 56, 64
x = torch.randn(n, H, H, Cc, device="cuda").to(torch.bfloat16)
w = (torch.randn(Cc, 3, 3, Cc, device="cuda") * 0.05).to(torch.bfloat16)
b = torch.zeros(Cc, device="cuda")
dz = torch.randn(n, H, H, Cc, device="cuda").to(torch.bfloat16)
sc = torch.randn(n, H, H, Cc, device="cuda").to(torch.bfloat16)
buf = (C.c_ulonglong * (4096 * 8))()
L = B.lib()
tiles = n * 28
names = ["prod wempty", "mma tempty", "mma wfull", "epi tfull", "epi efull", "epi bar1", "epi bar2", "mma total"]
for name, fn in [("fwd", lambda: B.dbg_conv_fwd(x, w, b, 1, 1, act=1)),
                 ("fwd+res", lambda: B.dbg_conv_fwd(x, w, b, 1, 1, act=1, res=sc)),
                 ("dgrad", lambda: B.dbg_conv_dgrad(dz, w, H, H, 1, 1, sc=sc, yact=x, mask_act=1))]:
    timing = hasattr(L, "adainf_dbg_wait_cycles")
    fn()
    torch.cuda.synchronize()
    if timing:
        L.adainf_dbg_wait_cycles(buf, 1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    fn()
    e1.record()
    torch.cuda.synchronize()
    if not timing:
        print(f"{name:8s} {e0.elapsed_time(e1)*1e3:7.1f} us", flush=True)
        continue
    L.adainf_dbg_wait_cycles(buf, 1)
    a = np.frombuffer(buf, dtype=np.uint64).reshape(4096, 8)[:148].astype(np.float64)
    per_tile = a.sum(0) / tiles
    print(f"{name:8s} {e0.elapsed_time(e1)*1e3:7.1f} us  per tile (cycles, summed over waiting warps): " +
          ", ".join(f"{nm} {v:.0f}" for nm, v in zip(names, per_tile)), flush=True)
