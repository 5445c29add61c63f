"""Diagnostic: forward closeness GPU vs oracle (final logits with all exits disabled) and single-conv
bf16 mismatch rates."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import numpy as np, torch
import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B, specs as S, synth
from parity import images, rel, to_cuda_bf16, gpu_infer_single
spec = S.resnet18_ee(in_hw=64)
p = synth.init_params(spec, seed=12)
xb, y, xf = images(spec, 12, 12)
orc = O.Model(spec).forward(p, xf)
g = gpu_infer_single(spec, p, xb, [2.0, 2.0, 2.0])
print("final logits rel per sample:", [f"{rel(g['logits'][i], orc['logits'][i,3]):.1e}" for i in range(12)])
print("embed rel:", rel(g["embed"], orc["pooled0"]))
# single conv mismatch rate
for (n, H, W, C, Co, K, s, pd) in [(4, 16, 16, 64, 64, 3, 1, 1), (2, 8, 8, 256, 256, 3, 1, 1), (2, 8, 8, 512, 512, 3, 1, 1)]:
    gen = torch.Generator().manual_seed(0)
    x = torch.randn(n, H, W, C, generator=gen).to(torch.bfloat16)
    w = (torch.randn(Co, K, K, C, generator=gen) / (K * K * C) ** 0.5).to(torch.bfloat16)
    b = torch.zeros(Co)
    out = B.dbg_conv_fwd(x.cuda(), w.cuda(), b.cuda(), s, pd, act=0, out_f32=True).cpu().numpy()
    out16 = B.dbg_conv_fwd(x.cuda(), w.cuda(), b.cuda(), s, pd, act=0).float().cpu().numpy()
    xs, ws = x.float().numpy(), w.float().numpy()
    mism, maxrel = [], 0
    for i in range(n):
        acc = O.conv_acc(xs[i], ws, s, pd)
        maxrel = max(maxrel, float(np.max(np.abs(out[i] - acc) / (np.abs(acc) + 1e-3))))
        mism.append(np.mean(O.bf16(acc) != out16[i]))
    print(f"conv C={C} Co={Co}: fp32 max rel err {maxrel:.2e}, bf16 mismatch rate {np.mean(mism):.2e}")
