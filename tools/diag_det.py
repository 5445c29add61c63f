"""Diagnostic (GPU box): detector score drift GPU vs oracle at 416x416 (all candidates via tau_det < 0)."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle as O  # noqa: E402
from paper_conf_sigcomm_shubhas23_b200 import binding as B  # noqa: E402
from paper_conf_sigcomm_shubhas23_b200 import specs as S  # noqa: E402
from paper_conf_sigcomm_shubhas23_b200 import synth  # noqa: E402

Bn, hw = 4, int(sys.argv[1]) if len(sys.argv) > 1 else 416
obj_bias = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0
spec = S.tiny_yolo_det(in_hw=hw)
A, NC = 3, 2
p = synth.det_head_params(spec, synth.init_params(spec, seed=21), obj_bias=obj_bias)
xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=41)
raw = O.Model(spec).forward(p, synth.bf16_bits_to_f32(xb), want_det=True)["det"]
G = raw.shape[1]
sig = lambda v: 1 / (1 + np.exp(-v.astype(np.float64)))
r5 = raw.reshape(Bn, G, G, A, 5 + NC)
scores = (sig(r5[..., 4]) * sig(r5[..., 5:].max(-1))).reshape(-1)
m = B.Model(spec, Bn, params=p)
app = B.App([m])
outs = B.alloc_outs(m, Bn, max_det=Bn * G * G * A)
app.infer(torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16), [-1.0], [outs])
torch.cuda.synchronize()
n = int(outs["n_det"].item())
g = outs["det_table"].cpu().numpy()[:n]
assert n == scores.size, (n, scores.size)
gs = g[:, 4].astype(np.float64)
d = np.abs(gs - scores)
res = {"hw": hw, "obj_bias": obj_bias, "n": n, "max_dscore": float(d.max()), "p99": float(np.quantile(d, 0.99)),
       "p50": float(np.median(d)), "frac_gt_1e-3": float((d > 1e-3).mean()),
       "score_q": np.quantile(scores, [0.01, 0.1, 0.5, 0.9, 0.99]).tolist(),
       "raw_absmax": float(np.abs(raw).max()), "raw_std": float(raw.std())}
print(json.dumps(res))
