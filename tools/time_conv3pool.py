"""Time conv3pool.cu at the C3 detector's layer shapes (512 frames; layers 1-3) through the debug entry point, with
algorithmic bytes (input read once + pooled output written) per launch: the kernel's HBM roofline."""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B

n = int(os.environ.get("N", "512"))
rows = []
for (H, C, Co, first) in [(416, 4, 16, True), (208, 16, 32, False), (104, 32, 64, False)]:
    x = (torch.randn(n, H, H, C, device="cuda") * 0.5).to(torch.bfloat16)
    w = (torch.randn(Co, 3, 3, C, device="cuda") * 0.1).to(torch.bfloat16)
    b = torch.zeros(Co, device="cuda")
    run = lambda: B.dbg_conv3_pool(x, w, b, act=2, first=first, cin_real=3 if first else C)
    y = run()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5):
        run()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    by = n * H * H * (3 if first else C) * 2 + y.numel() * 2
    rows.append({"H": H, "cin": C, "cout": Co, "first": first, "ms": round(ms, 3), "gbs": round(by / ms / 1e6, 1)})
    del x, y
print(json.dumps(rows))
