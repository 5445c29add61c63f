"""Barrier-wait attribution of the layer-1 weight-gradient window kernel (conv_wgrad_win_tma_kernel) from a
-DADAINF_TIMING build (see tools/time_waits.py).  Slots: 0 producer empty, 1 MMA tempty, 2 MMA full,
3 epilogue tfull, 4 column-sum warps full; printed per K-block (summed over the waiting warps)."""
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
x = torch.randn(n, 56, 56, 64, device="cuda").to(torch.bfloat16)
dz = torch.randn(n, 56, 56, 64, device="cuda").to(torch.bfloat16)
L = B.lib()
buf = (C.c_ulonglong * (4096 * 8))()
fn = lambda: B.dbg_conv_wgrad(x, dz, 3, 3, 1, 1)
fn()
torch.cuda.synchronize()
L.adainf_dbg_wait_cycles(buf, 1)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
fn()
e1.record()
torch.cuda.synchronize()
L.adainf_dbg_wait_cycles(buf, 1)
a = np.frombuffer(buf, dtype=np.uint64).reshape(4096, 8)[:148].astype(np.float64)
nkb = n * 14  # K-blocks of 4 rows x 64 pitch per image (56 rows)
print(f"wgrad {e0.elapsed_time(e1)*1e3:.1f} us; per K-block (cycles summed over waiting warps): " +
      ", ".join(f"slot{i} {v:.0f}" for i, v in enumerate(a.sum(0) / nkb)), flush=True)
