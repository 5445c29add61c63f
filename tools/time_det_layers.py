"""Time every conv of the TinyYOLOv3-like detector (BASELINE config 3) at 512 frames of 416x416 through the debug
conv entry point (CUDA events), with algorithmic FLOPs and bytes per layer: which layers bound the C3 DAG."""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S

n = int(os.environ.get("N", "512"))
spec = S.tiny_yolo_det()
H = W = spec["in_h"]
C = 8
rows = []
for o in spec["ops"]:
    if o["kind"] == "maxpool":
        H = (H + 2 * o["pad"] - o["kh"]) // o["stride"] + 1
        W = (W + 2 * o["pad"] - o["kw"]) // o["stride"] + 1
        continue
    if o["kind"] != "conv":
        continue
    x = torch.randn(n, H, W, C, device="cuda").to(torch.bfloat16)
    Co = o["cout"] if o["cout"] % 8 == 0 else 24
    w = (torch.randn(Co, o["kh"], o["kw"], C, device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(Co, device="cuda")
    f32 = o["cout"] % 8 != 0

    def run():
        return B.dbg_conv_fwd(x, w, b, o["stride"], o["pad"], act=o["act"], out_f32=f32)

    y = run()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        run()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    Ho, Wo = y.shape[1], y.shape[2]
    fl = 2.0 * n * Ho * Wo * Co * o["kh"] * o["kw"] * C
    by = x.numel() * 2 + y.numel() * y.element_size()
    rows.append({"H": H, "cin": C, "cout": Co, "k": o["kh"], "ms": round(ms, 3), "tflops": round(fl / ms / 1e9, 1),
                 "gbs": round(by / ms / 1e6, 1)})
    del x, y
    H, W, C = Ho, Wo, Co
print(json.dumps(rows, indent=0))
