"""Diagnostic: MobileNetV2-EE retraining gradients, GPU vs oracle per tensor, next to the oracle's own response to
20 one-ulp input flips and to the exact (fp64, no bf16 storage) gradient."""
import sys
sys.path[:0] = [".", "tests"]
import numpy as np
import torch
import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B, specs as S, synth
from parity import bn_folded_params, images, rel, to_cuda_bf16

spec = S.mobilenetv2_ee(in_hw=64, width=0.5)
n = 16
p = synth.init_params(spec, seed=72)
xb, y, xf = images(spec, n, 72)
p = bn_folded_params(spec, p, xf)
p = synth.spread_exit_heads(spec, p, O.Model(spec).forward(p, xf)["logits"])
m_o = O.Model(spec)
_, _, g_o, loss_o = m_o.retrain_step(p, np.zeros_like(p), xf, y, lr=0.01, mu=0.9)
rng = np.random.default_rng(0)
x2 = xb.copy().view(np.uint16)
x2.reshape(-1)[rng.choice(x2.size, 20, replace=False)] ^= 1
_, _, g_s, _ = m_o.retrain_step(p, np.zeros_like(p), synth.bf16_bits_to_f32(x2.view(xb.dtype)), y, lr=0.01, mu=0.9)
g_x = m_o.grad_exact(p.astype(np.float64), xf.astype(np.float64), y)
m = B.Model(spec, n, params=p, momentum=0.9)
m.retrain_step(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), lr=0.01)
torch.cuda.synchronize()
g_g = m.get_grads()
print("loss", loss_o)
print(f"{'tensor':>14} {'gpu-vs-or':>10} {'or-sens':>10} {'or-vs-exact':>12} {'gpu-vs-exact':>12}")
for kind, i, off, shp in S.param_segments(spec):
    c = int(np.prod(shp))
    sl = slice(off, off + c)
    print(f"{kind:>8} {i:>5} {rel(g_g[sl], g_o[sl]):10.2e} {rel(g_s[sl], g_o[sl]):10.2e} {rel(g_o[sl], g_x[sl]):12.2e} "
          f"{rel(g_g[sl], g_x[sl]):12.2e}")
