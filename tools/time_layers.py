"""Time every distinct ResNet-18 conv shape (fwd + dgrad + wgrad) at the retraining batch under each dispatch mode
(ADAINF window mode: 0 = generic implicit GEMM only, 1 = default routing).  CUDA events, 5 reps."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
if os.environ.get("ADAINF_LIB"):  # A/B against another build
    B.LIB_PATH = os.environ["ADAINF_LIB"]

n = int(os.environ.get("N", "1024"))
modes = [int(m) for m in os.environ.get("MODES", "0,1").split(",")]
# (H_in, Cin, Cout, K, stride)
shapes = [(56, 64, 64, 3, 1), (56, 64, 128, 3, 2), (56, 64, 128, 1, 2), (28, 128, 128, 3, 1),
          (28, 128, 256, 3, 2), (28, 128, 256, 1, 2), (14, 256, 256, 3, 1), (14, 256, 512, 3, 2),
          (14, 256, 512, 1, 2), (7, 512, 512, 3, 1)]
sel = os.environ.get("SHAPES")
if sel:
    shapes = [shapes[int(i)] for i in sel.split(",")]


def t(fn, reps=int(os.environ.get("REPS", "5"))):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


for (H, C, Co, K, s) in shapes:
    p = K // 2
    Ho = (H + 2 * p - K) // s + 1
    x = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
    w = (torch.randn(Co, K, K, C, device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(Co, device="cuda")
    dz = torch.randn(n, Ho, Ho, Co, device="cuda").to(torch.bfloat16)
    sc = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
    fl = 2 * n * Ho * Ho * Co * K * K * C
    for m in modes:
        B.dbg_set_win_mode(m)
        for name, fn in [("fwd", lambda: B.dbg_conv_fwd(x, w, b, s, p, act=1)),
                         ("dgrad", lambda: B.dbg_conv_dgrad(dz, w, H, H, s, p, sc=sc, yact=x, mask_act=1)),
                         ("dgrad-nosc", lambda: B.dbg_conv_dgrad(dz, w, H, H, s, p, yact=x, mask_act=1)),
                         ("wgrad", lambda: B.dbg_conv_wgrad(x, dz, K, K, s, p))]:
            ms = t(fn)
            print(f"H={H:3d} {C:3d}->{Co:3d} k{K} s{s} mode={m} {name:6s} {ms*1e3:8.1f} us "
                  f"{fl/ms/1e9:7.1f} TFLOP/s", flush=True)
B.dbg_set_win_mode(1)
