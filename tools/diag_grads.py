"""Diagnostic: per-tensor gradient rel errors GPU vs oracle (bf16 storage) and oracle bf16 vs exact."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import numpy as np, torch
import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B, specs as S, synth
from parity import images, rel, to_cuda_bf16
hw = int(sys.argv[1]) if len(sys.argv) > 1 else 64
n = int(sys.argv[2]) if len(sys.argv) > 2 else 12
spec = S.resnet18_ee(in_hw=hw)
p = synth.init_params(spec, seed=12)
xb, y, xf = images(spec, n, 12)
om = O.Model(spec)
p1, v1, g_o, loss_o = om.retrain_step(p, np.zeros_like(p), xf, y, n_global=48, lr=0.01)
ge = om.grad_exact(synth.round_bf16(p).astype(np.float64), xf, y, n_global=48)
m = B.Model(spec, n, params=p)
m.retrain_step(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), n_global=48, lr=0.01)
torch.cuda.synchronize()
g = m.get_grads()
for kind, i, off, shp in S.param_segments(spec):
    k = int(np.prod(shp))
    print(f"{kind:7s} op{i:3d} {str(shp):22s} gpu-vs-oracle {rel(g[off:off+k], g_o[off:off+k]):.2e}  oracle-bf16-vs-exact {rel(g_o[off:off+k], ge[off:off+k]):.2e}  gpu-vs-exact {rel(g[off:off+k], ge[off:off+k]):.2e}")
