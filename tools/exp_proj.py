"""Time the 1x1/2 projection forward (and a 3x3/2 for contrast) under ADAINF_EXP flags given in argv."""
import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
n = int(os.environ.get("N", "1024"))
for (H, C, Co, K, s) in [(56, 64, 128, 1, 2), (28, 128, 256, 1, 2), (56, 64, 128, 3, 2), (56, 64, 128, 1, 1)]:
    p = K // 2
    Ho = (H + 2 * p - K) // s + 1
    x = torch.randn(n, H, H, C, device="cuda").to(torch.bfloat16)
    w = (torch.randn(Co, K, K, C, device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(Co, device="cuda")
    fn = lambda: B.dbg_conv_fwd(x, w, b, s, p, act=0)
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5): fn()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    by = n * Ho * Ho * (C + Co) * 2
    print(f"EXP={os.environ.get('ADAINF_EXP','0')} H={H} {C}->{Co} k{K} s{s}: {ms*1e3:.1f} us  {by/ms/1e6:.0f} GB/s(min bytes)", flush=True)
