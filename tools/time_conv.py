"""Time single conv launches (fwd/dgrad/wgrad) with CUDA events at ResNet-18 training shapes."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
n = int(os.environ.get("N", "1024"))
modes = [int(m) for m in os.environ.get("MODES", "0,1").split(",")]
shapes = [(56, 64, 64), (28, 128, 128), (14, 256, 256), (7, 512, 512)]
for (H, C, Co) in (shapes if os.environ.get("FWD", "1") == "1" else []):
    x = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
    w = (torch.randn(Co, 3, 3, C, device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(Co, device="cuda")
    dz = torch.randn(n, H, H, Co, device="cuda").to(torch.bfloat16)
    fl = 2 * n * H * H * Co * 9 * C
    for m in modes:
        B.dbg_set_win_mode(m)
        for name, fn in [("fwd", lambda: B.dbg_conv_fwd(x, w, b, 1, 1, act=1)),
                         ("dgrad", lambda: B.dbg_conv_dgrad(dz, w, H, H, 1, 1))]:
            fn(); torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(5): fn()
            e1.record(); torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / 5
            print(f"H={H:3d} C={C:3d} mode={m} {name:6s} {ms*1e3:8.1f} us {fl/ms/1e9:7.1f} TFLOP/s", flush=True)
B.dbg_set_win_mode(1)
# wgrad timing
if os.environ.get("WGRAD", "1") == "1":
    wshapes = [(56, 64, 64, 3, 1), (28, 128, 128, 3, 1), (14, 256, 256, 3, 1), (7, 512, 512, 3, 1),
               (56, 64, 128, 3, 2), (28, 128, 256, 3, 2), (14, 256, 512, 3, 2),
               (56, 64, 128, 1, 2), (28, 128, 256, 1, 2), (14, 256, 512, 1, 2)]
    for (H, C, Co, K, s) in wshapes:
        Ho = (H + 2 * (K // 2) - K) // s + 1
        x = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
        dz = torch.randn(n, Ho, Ho, Co, device="cuda").to(torch.bfloat16)
        fl = 2 * n * Ho * Ho * Co * K * K * C
        for m in modes:
            B.dbg_set_win_mode(m)
            B.dbg_conv_wgrad(x, dz, K, K, s, K // 2); torch.cuda.synchronize()
            B.prof_enable(True); B.prof_reset()
            for _ in range(5): B.dbg_conv_wgrad(x, dz, K, K, s, K // 2)
            torch.cuda.synchronize()
            q = B.prof_query(); B.prof_enable(False)
            ms = q["conv_wgrad"][1] / 5
            red = q.get("wgrad_reduce", (0, 0.0))[1] / 5
            cs = q.get("bias_colsum", (0, 0.0))[1] / 5
            print(f"H={H:3d} C={C:3d} Co={Co:3d} K={K} s={s} mode={m} wgrad {ms*1e3:8.1f} us {fl/ms/1e9:7.1f} TFLOP/s"
                  f"  reduce {red*1e3:6.1f} us  colsum {cs*1e3:6.1f} us", flush=True)
    B.dbg_set_win_mode(1)
