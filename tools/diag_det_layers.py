"""Diagnostic (GPU box): per-layer rounding agreement of the detector's convs.  Each layer's bf16 input is
produced by an fp64 torch emulation of the oracle's rounding points (conv fp64 -> fp32 -> +b fp32 -> leaky
(0.1f*x fp32) -> bf16); the same input runs through the GPU conv kernel (adainf_dbg_conv_fwd); reported per
layer: fraction of outputs whose bf16 value differs, and the max |diff| in bf16 ulps; plus the end-to-end raw
head error of the full GPU model vs the oracle.  usage: python tools/diag_det_layers.py [hw] [frames]"""
import json
import sys

import numpy as np
import torch
import torch.nn.functional as F

sys.path.insert(0, ".")
from paper_conf_sigcomm_shubhas23_b200 import binding as B  # noqa: E402
from paper_conf_sigcomm_shubhas23_b200 import specs as S  # noqa: E402
from paper_conf_sigcomm_shubhas23_b200 import synth  # noqa: E402

hw = int(sys.argv[1]) if len(sys.argv) > 1 else 416
nf = int(sys.argv[2]) if len(sys.argv) > 2 else 2
spec = S.tiny_yolo_det(in_hw=hw)
p = synth.det_head_params(spec, synth.init_params(spec, seed=21), obj_bias=0.0)
xb, _ = synth.drifted_images(nf, hw, hw, 3, seed=41)
segs = {(k, i): (off, shp) for k, i, off, shp in S.param_segments(spec)}


def seg(kind, i):
    off, shp = segs[(kind, i)]
    return p[off:off + int(np.prod(shp))].reshape(shp)


def R(t):
    return t.float().to(torch.bfloat16).double()


cur = torch.from_numpy(synth.bf16_bits_to_f32(xb).astype(np.float64))  # NHWC
rows = []
ops = spec["ops"]
for i, o in enumerate(ops):
    if o["kind"] == "maxpool":
        cur = F.max_pool2d(cur.permute(0, 3, 1, 2), o["kh"], o["stride"], o["pad"]).permute(0, 2, 3, 1)
        continue
    if o["kind"] != "conv":
        continue
    w = seg("conv_w", i)  # [Co][kh][kw][Cin]
    b = seg("conv_b", i)
    wr = R(torch.from_numpy(w.astype(np.float64)))
    acc = F.conv2d(cur.permute(0, 3, 1, 2), wr.permute(0, 3, 1, 2), stride=o["stride"], padding=o["pad"])
    v = acc.float().double() + torch.from_numpy(b.astype(np.float64))[None, :, None, None]
    v = v.float().double()
    if o["act"] == 2:
        v = torch.where(v > 0, v, (v.float() * torch.tensor(0.1, dtype=torch.float32)).double())
    fp32_out = i + 1 < len(ops) and ops[i + 1]["kind"] == "det_head"
    ref = (v.float().double() if fp32_out else R(v)).permute(0, 2, 3, 1)
    # GPU: same bf16 input (channels padded to a multiple of 8)
    Cin = cur.shape[3]
    Cp = (Cin + 7) // 8 * 8
    xin = torch.zeros(cur.shape[:3] + (Cp,), dtype=torch.float64)
    xin[..., :Cin] = cur
    wp = np.zeros(w.shape[:3] + (Cp,), np.float32)
    wp[..., :Cin] = w
    xg = xin.float().to(torch.bfloat16).cuda()
    wg = torch.from_numpy(wp).to(torch.bfloat16).cuda()
    bg = torch.from_numpy(b.astype(np.float32)).cuda()
    out = B.dbg_conv_fwd(xg, wg, bg, o["stride"], o["pad"], act=o["act"], out_f32=fp32_out)
    torch.cuda.synchronize()
    g = out.double().cpu()
    diff = (g != ref)
    rel = ((g - ref).abs() / ref.abs().clamp_min(1e-30))
    rows.append({"layer": i, "k": f"{o['kh']}x{o['kw']}", "cin": Cin, "cout": o["cout"], "K": Cin * o["kh"] * o["kw"],
                 "frac_diff": float(diff.double().mean()), "max_rel_of_diffs": float(rel[diff].max()) if diff.any() else 0.0,
                 "ref_absmax": float(ref.abs().max()), "ref_std": float(ref.std())})
    cur = ref
print(json.dumps(rows, indent=0))
