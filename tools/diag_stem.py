"""Diagnose the stem weight gradient: map each (tap, s2d channel) entry of the kernel's dW to the best
matching reference entry (correlation over the 64 output channels)."""
import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
from paper_conf_sigcomm_shubhas23_b200 import binding as B
n, H, W, cin = [int(v) for v in os.environ.get("CASE", "2,32,32,4").split(",")]
g = torch.Generator().manual_seed(4)
x = torch.randn(n, H, W, cin, generator=g).to(torch.bfloat16).cuda()
dz = torch.randn(n, H // 2, W // 2, 64, generator=g).to(torch.bfloat16).cuda()
dw, db = B.dbg_stem_wgrad(x, dz)
ref = torch.nn.grad.conv2d_weight(x.float().permute(0, 3, 1, 2), (64, cin, 7, 7), dz.float().permute(0, 3, 1, 2),
                                  stride=2, padding=3).permute(0, 2, 3, 1)
print("db rel", float((db - dz.float().sum((0, 1, 2))).norm() / db.norm()))
def s2d(w):
    out = {}
    for t in range(16):
        ah, aw = t // 4 - 2, t % 4 - 2
        for ch in range(16):
            bh, bw, c = ch >> 3, (ch >> 2) & 1, ch & 3
            kh, kw = 2 * ah + bh + 3, 2 * aw + bw + 3
            if 0 <= kh < 7 and 0 <= kw < 7 and c < cin:
                out[(t, ch)] = w[:, kh, kw, c]
    return out
A, R = s2d(dw), s2d(ref)
keys = list(R.keys())
Rm = torch.stack([R[k] for k in keys])
Rn = Rm / Rm.norm(dim=1, keepdim=True)
ok = 0
for k in sorted(A.keys()):
    v = A[k] / A[k].norm().clamp_min(1e-9)
    cor = Rn @ v
    j = int(cor.argmax())
    if keys[j] == k and float(cor[j]) > 0.999:
        ok += 1
    else:
        print("ours", k, "-> ref", keys[j], "corr %.4f" % float(cor[j]), "norm ratio %.3f" % float(A[k].norm() / R[keys[j]].norm()))
print("matching", ok, "of", len(A))
rel = float((dw - ref).norm() / ref.norm())
print("dw rel", rel)
err = (dw - ref).abs()
idx = torch.nonzero(err > 1e-3 * ref.abs().max())
print("entries off:", idx.shape[0], "of", ref.numel())
if idx.shape[0]:
    print("kh,kw,c of first offenders:", idx[:20, 1:].tolist())
