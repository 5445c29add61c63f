"""Diagnostic: MobileNetV2-EE GPU vs oracle logits relative error per exit (tau truncation at each exit)."""
import sys
import numpy as np
sys.path.insert(0, "tests")
sys.path.insert(0, ".")
import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import specs as S, synth
from parity import bn_folded_params, gpu_infer_single, images, rel

for hw, width, Bn, spread in [(64, 0.5, 24, True), (64, 0.5, 24, False), (96, 1.0, 12, True)]:
    spec = S.mobilenetv2_ee(in_hw=hw, width=width)
    p = synth.init_params(spec, seed=71)
    xb, _, xf = images(spec, Bn, 71)
    p = bn_folded_params(spec, p, xf)
    if spread:
        p = synth.spread_exit_heads(spec, p, O.Model(spec).forward(p, xf)["logits"])
    orc = O.Model(spec).forward(p, xf)
    E = orc["conf"].shape[1]
    print(f"hw {hw} width {width} spread {spread}")
    for k in range(E):
        taus = [2.0] * (E - 1)
        if k < E - 1:
            taus[k] = 0.0
        g = gpu_infer_single(spec, p, xb, taus)
        assert (g["exit_id"] == k).all()
        r = [rel(g["logits"][n], orc["logits"][n, k]) for n in range(Bn)]
        dc = np.abs(g["conf"] - orc["conf"][:, k]).max()
        print(f"  exit {k}: rel logits median {np.median(r):.2e} max {max(r):.2e}  max dconf {dc:.2e}")
    print("  embed rel", rel(g["embed"], orc["pooled0"]))
