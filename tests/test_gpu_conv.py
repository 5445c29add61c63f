"""Per-kernel GPU parity of the tcgen05 implicit-GEMM conv (fwd / dgrad / wgrad) through the C-ABI
(include/adainf_debug.h).  Small shapes are checked against the oracle's direct-loop conv (fp64
accumulation); all shapes against torch fp32 on the same bf16 operands.  Shapes span several M/N tiles,
ragged tails, stride-2 phases, 1x1 / 3x3 / 7x7 kernels and every BN variant."""
import numpy as np
import pytest
import torch

from paper_conf_sigcomm_shubhas23_b200 import binding as B

pytestmark = pytest.mark.gpu

FWD_CASES = [  # n, H, W, C, Co, K, s, p
    (2, 9, 7, 8, 32, 3, 1, 1),
    (3, 14, 14, 64, 64, 3, 1, 1),
    (2, 15, 13, 64, 128, 3, 2, 1),
    (2, 8, 8, 128, 256, 1, 2, 0),
    (1, 21, 20, 8, 64, 7, 2, 3),
    (2, 7, 7, 256, 512, 3, 1, 1),
    (5, 13, 13, 32, 24, 1, 1, 0),
    (2, 23, 21, 4, 64, 7, 2, 3),   # 4-channel (8-byte pixel) stem path
    (3, 12, 12, 4, 32, 3, 1, 1),
]


def _rel(a, b):
    a, b = a.double(), b.double()
    return float((a - b).norm() / b.norm().clamp_min(1e-30))


def _mk(case, seed):
    n, H, W, C, Co, K, s, p = case
    g = torch.Generator(device="cpu").manual_seed(seed)
    x = torch.randn(n, H, W, C, generator=g).to(torch.bfloat16).cuda()
    w = (torch.randn(Co, K, K, C, generator=g) * (2.0 / (K * K * C)) ** 0.5).to(torch.bfloat16).cuda()
    b = (torch.randn(Co, generator=g) * 0.1).cuda()
    return x, w, b


def _ref_fwd(x, w, b, s, p):
    return torch.nn.functional.conv2d(x.float().permute(0, 3, 1, 2), w.float().permute(0, 3, 1, 2), b, stride=s,
                                      padding=p).permute(0, 2, 3, 1)


@pytest.mark.parametrize("case", FWD_CASES)
@pytest.mark.parametrize("act", [0, 1, 2])
def test_conv_fwd_vs_torch(case, act):
    n, H, W, C, Co, K, s, p = case
    x, w, b = _mk(case, 1)
    ref = _ref_fwd(x, w, b, s, p)
    if act == 1:
        ref = torch.relu(ref)
    elif act == 2:
        ref = torch.where(ref > 0, ref, 0.1 * ref)
    out = B.dbg_conv_fwd(x, w, b, s, p, act=act)
    torch.cuda.synchronize()
    assert out.shape == ref.shape
    assert _rel(out.float(), ref) < 8e-3


def test_conv_fwd_residual_and_f32_out():
    case = (3, 14, 14, 64, 64, 3, 1, 1)
    x, w, b = _mk(case, 2)
    res = torch.randn(3, 14, 14, 64).to(torch.bfloat16).cuda()
    ref = torch.relu(_ref_fwd(x, w, b, 1, 1) + res.float())
    out = B.dbg_conv_fwd(x, w, b, 1, 1, act=1, res=res)
    assert _rel(out.float(), ref) < 8e-3
    case = (4, 13, 13, 64, 21, 1, 1, 0)
    x, w, b = _mk(case, 3)
    out = B.dbg_conv_fwd(x, w, b, 1, 0, act=0, out_f32=True)
    assert out.dtype == torch.float32
    assert _rel(out, _ref_fwd(x, w, b, 1, 0)) < 1e-4


def test_conv_fwd_vs_oracle_exact_small():
    """fp32 accumulate vs the oracle's fp64 sum, then bf16 rounding on both: nearly all equal."""
    import oracle as O
    case = (2, 9, 7, 16, 32, 3, 2, 1)
    x, w, b = _mk(case, 4)
    out = B.dbg_conv_fwd(x, w, b, 2, 1, act=0).float().cpu().numpy()
    xs, ws, bs = x.float().cpu().numpy(), w.float().cpu().numpy(), b.cpu().numpy()
    for i in range(2):
        acc = O.conv_acc(xs[i], ws, 2, 1) + bs
        ref = O.bf16(acc.astype(np.float32))
        mism = np.mean(ref != out[i])
        assert mism < 0.01, mism
        np.testing.assert_allclose(out[i], ref, rtol=1e-2, atol=1e-2)


@pytest.mark.parametrize("case", [c for c in FWD_CASES if c[4] % 8 == 0 and c[3] % 8 == 0])
def test_conv_dgrad_vs_torch(case):
    n, H, W, C, Co, K, s, p = case
    x, w, b = _mk(case, 5)
    Ho, Wo = (H + 2 * p - K) // s + 1, (W + 2 * p - K) // s + 1
    dz = torch.randn(n, Ho, Wo, Co).to(torch.bfloat16).cuda()
    ref = torch.nn.grad.conv2d_input((n, C, H, W), w.float().permute(0, 3, 1, 2), dz.float().permute(0, 3, 1, 2),
                                     stride=s, padding=p).permute(0, 2, 3, 1)
    dx = B.dbg_conv_dgrad(dz, w, H, W, s, p)
    torch.cuda.synchronize()
    assert _rel(dx.float(), ref) < 8e-3


# stride-2 3x3 layers take the sub-pixel dgrad (one GEMM over the dZ grid, N = 4 * Cin): ResNet shapes at small
# batch, odd spatial sizes (the last output row / column phase is dropped), a ragged last M tile
SP_CASES = [(3, 56, 56, 64, 128, 3, 2, 1), (2, 28, 28, 128, 256, 3, 2, 1), (2, 14, 14, 256, 512, 3, 2, 1),
            (3, 7, 9, 128, 64, 3, 2, 1), (1, 13, 11, 64, 192, 3, 2, 1)]


@pytest.mark.parametrize("case", SP_CASES)
def test_conv_dgrad_subpixel_vs_torch(case):
    n, H, W, C, Co, K, s, p = case
    x, w, b = _mk(case, 7)
    Ho, Wo = (H + 2 * p - K) // s + 1, (W + 2 * p - K) // s + 1
    g = torch.Generator(device="cpu").manual_seed(8)
    dz = torch.randn(n, Ho, Wo, Co, generator=g).to(torch.bfloat16).cuda()
    bc = torch.randn(n, C, generator=g).cuda() * 0.01
    sc = torch.randn(n, H, W, C, generator=g).to(torch.bfloat16).cuda()
    y = torch.randn(n, H, W, C, generator=g).to(torch.bfloat16).cuda()
    ref = torch.nn.grad.conv2d_input((n, C, H, W), w.float().permute(0, 3, 1, 2), dz.float().permute(0, 3, 1, 2),
                                     stride=s, padding=p).permute(0, 2, 3, 1)
    dx = B.dbg_conv_dgrad(dz, w, H, W, s, p)
    torch.cuda.synchronize()
    assert _rel(dx.float(), ref) < 8e-3
    ref2 = (ref + bc[:, None, None, :] + sc.float()) * (y.float() > 0)
    dx2 = B.dbg_conv_dgrad(dz, w, H, W, s, p, bcast=bc, sc=sc, yact=y, mask_act=1)
    assert _rel(dx2.float(), ref2) < 8e-3


def test_conv_dgrad_epilogue_terms():
    case = (2, 14, 14, 64, 128, 3, 2, 1)
    n, H, W, C, Co, K, s, p = case
    x, w, b = _mk(case, 6)
    dz = torch.randn(n, 7, 7, Co).to(torch.bfloat16).cuda()
    bc = torch.randn(n, C).cuda() * 0.01
    sc = torch.randn(n, H, W, C).to(torch.bfloat16).cuda()
    y = torch.randn(n, H, W, C).to(torch.bfloat16).cuda()
    ref = torch.nn.grad.conv2d_input((n, C, H, W), w.float().permute(0, 3, 1, 2), dz.float().permute(0, 3, 1, 2),
                                     stride=s, padding=p).permute(0, 2, 3, 1)
    ref = (ref + bc[:, None, None, :] + sc.float()) * (y.float() > 0)
    dx = B.dbg_conv_dgrad(dz, w, H, W, s, p, bcast=bc, sc=sc, yact=y, mask_act=1)
    assert _rel(dx.float(), ref) < 8e-3


# extra wgrad shapes for the TMA path: Wo up to 64 (Wp=64, one row per K-block), odd channel blocks
# (a half-empty last M tile), stride-2 3x3 and 1x1 with ragged spatial tails
WG_CASES = [(3, 56, 56, 64, 64, 3, 1, 1), (2, 28, 28, 128, 128, 3, 1, 1), (4, 29, 27, 192, 64, 3, 1, 1),
            (2, 17, 17, 64, 128, 1, 2, 0), (3, 31, 29, 64, 128, 3, 2, 1), (2, 33, 64, 64, 256, 3, 1, 1)]


@pytest.mark.parametrize("case", [c for c in FWD_CASES if c[4] % 8 == 0] + WG_CASES)
def test_conv_wgrad_vs_torch(case):
    n, H, W, C, Co, K, s, p = case
    x, w, b = _mk(case, 7)
    Ho, Wo = (H + 2 * p - K) // s + 1, (W + 2 * p - K) // s + 1
    dz = torch.randn(n, Ho, Wo, Co).to(torch.bfloat16).cuda()
    ref = torch.nn.grad.conv2d_weight(x.float().permute(0, 3, 1, 2), (Co, C, K, K), dz.float().permute(0, 3, 1, 2),
                                      stride=s, padding=p).permute(0, 2, 3, 1)
    dw, db = B.dbg_conv_wgrad(x, dz, K, K, s, p)
    torch.cuda.synchronize()
    assert _rel(dw, ref) < 1e-4
    assert _rel(db, dz.float().sum(dim=(0, 1, 2))) < 1e-5
    # deterministic: same bits on a second run
    dw2, db2 = B.dbg_conv_wgrad(x, dz, K, K, s, p)
    assert torch.equal(dw, dw2) and torch.equal(db, db2)


WIN_CASES = [(2, 14, 14, 64, 64), (3, 7, 7, 128, 256), (2, 28, 28, 64, 128), (1, 56, 56, 64, 64), (5, 9, 11, 64, 64),
             (2, 14, 14, 256, 256), (3, 28, 28, 128, 128), (2, 12, 20, 128, 128), (2, 9, 13, 128, 256),
             # odd tiles per image (W = 20 -> pitch 32, 4 rows per tile, 5 tiles): the last tile pair of the
             # 64-channel kernel's pair mode has one tile inside the image
             (3, 20, 20, 64, 64)]


@pytest.mark.parametrize("mode", [1, 2])
@pytest.mark.parametrize("case", WIN_CASES)
def test_window_kernel_fwd_dgrad(case, mode):
    """Window implicit GEMM (stride-1 3x3) vs torch: tap A operands are row-shifted views of one window
    (mode 2 forces the window kernel for every eligible fwd/dgrad shape; the default routes by size)."""
    n, H, W, C, Co = case
    B.dbg_set_win_mode(mode)
    try:
        x, w, b = _mk((n, H, W, C, Co, 3, 1, 1), 11)
        res = torch.randn(n, H, W, Co).to(torch.bfloat16).cuda()
        ref = torch.relu(_ref_fwd(x, w, b, 1, 1) + res.float())
        out = B.dbg_conv_fwd(x, w, b, 1, 1, act=1, res=res)
        torch.cuda.synchronize()
        assert _rel(out.float(), ref) < 8e-3, ("fwd", mode)
        dz = torch.randn(n, H, W, Co).to(torch.bfloat16).cuda()
        y = torch.randn(n, H, W, C).to(torch.bfloat16).cuda()
        bc = torch.randn(n, C).cuda() * 0.01
        refd = torch.nn.grad.conv2d_input((n, C, H, W), w.float().permute(0, 3, 1, 2), dz.float().permute(0, 3, 1, 2),
                                          stride=1, padding=1).permute(0, 2, 3, 1)
        refd = (refd + bc[:, None, None, :]) * (y.float() > 0)
        dx = B.dbg_conv_dgrad(dz, w, H, W, 1, 1, bcast=bc, yact=y, mask_act=1)
        torch.cuda.synchronize()
        assert _rel(dx.float(), refd) < 8e-3, ("dgrad", mode)
    finally:
        B.dbg_set_win_mode(1)


@pytest.mark.parametrize("mode", [1, 5, 6, 7])
@pytest.mark.parametrize("case", WIN_CASES)
def test_window_wgrad(case, mode):
    """Stride-1 3x3 weight gradient through each routing: 1 = default (TMA window from 14 columns up, else
    TMA generic), 7 = TMA window forced (nine taps from one X window), 6 = TMA generic (one tap pair per
    M tile), 5 = no TMA (cp.async window for 64x64, else generic).  The bias gradient is fused into the
    TMA kernels and a separate pass otherwise."""
    n, H, W, C, Co = case
    B.dbg_set_win_mode(mode)
    try:
        x, _, _ = _mk((n, H, W, C, Co, 3, 1, 1), 12)
        dz = torch.randn(n, H, W, Co).to(torch.bfloat16).cuda()
        ref = torch.nn.grad.conv2d_weight(x.float().permute(0, 3, 1, 2), (Co, C, 3, 3), dz.float().permute(0, 3, 1, 2),
                                          stride=1, padding=1).permute(0, 2, 3, 1)
        dw, db = B.dbg_conv_wgrad(x, dz, 3, 3, 1, 1)
        torch.cuda.synchronize()
        assert _rel(dw, ref) < 1e-4, mode
        assert _rel(db, dz.float().sum(dim=(0, 1, 2))) < 1e-5
    finally:
        B.dbg_set_win_mode(1)


@pytest.mark.parametrize("H,C,Co", [(28, 128, 128), (14, 256, 256), (12, 128, 128)])
def test_wide_tile_kernels_vs_torch(H, C, Co):
    """The wide-tile conv kernels at small sizes (ADAINF_NARROW=0 keeps BN = Cout so they are reached):
    generic (ADAINF_DUALM=0), dual-M (two 128-row tiles sharing the weight tile, BN = 128) and the CTA pair
    (tcgen05.mma.cta_group::2, ADAINF_PAIR=1), forward (+ residual, ReLU) and stride-1 dgrad (+ shortcut term,
    ReLU mask), each against torch, and bit-identical to each other (same K order per output row)."""
    import os, subprocess, sys
    code = f"""
import sys, torch
sys.path.insert(0, {os.path.dirname(os.path.dirname(os.path.abspath(__file__)))!r})
from paper_conf_sigcomm_shubhas23_b200 import binding as B
g = torch.Generator().manual_seed(0)
n = 5  # ragged last tile
x = torch.randn(n, {H}, {H}, {C}, generator=g).to(torch.bfloat16).cuda()
w = (torch.randn({Co}, 3, 3, {C}, generator=g) * 0.05).to(torch.bfloat16).cuda()
b = (torch.randn({Co}, generator=g) * 0.1).cuda()
res = torch.randn(n, {H}, {H}, {Co}, generator=g).to(torch.bfloat16).cuda()
dz = torch.randn(n, {H}, {H}, {Co}, generator=g).to(torch.bfloat16).cuda()
sc = torch.randn(n, {H}, {H}, {C}, generator=g).to(torch.bfloat16).cuda()
y = B.dbg_conv_fwd(x, w, b, 1, 1, act=1, res=res)
dx = B.dbg_conv_dgrad(dz, w, {H}, {H}, 1, 1, sc=sc, yact=x, mask_act=1)
torch.cuda.synchronize()
torch.save({{"y": y.cpu(), "dx": dx.cpu()}}, sys.argv[1])
"""
    variants = {"generic": {"ADAINF_DUALM": "0", "ADAINF_PAIR": "0"}, "dualm": {"ADAINF_DUALM": "1", "ADAINF_PAIR": "0"},
                "pair": {"ADAINF_DUALM": "0", "ADAINF_PAIR": "1"}}
    outs = {}
    for name, extra in variants.items():
        path = f"/tmp/wide_{name}_{H}_{C}.pt"
        env = dict(os.environ, ADAINF_NARROW="0", **extra)
        r = subprocess.run([sys.executable, "-c", code, path], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        outs[name] = torch.load(path)
    g = torch.Generator().manual_seed(0)
    n = 5
    x = torch.randn(n, H, H, C, generator=g).to(torch.bfloat16)
    w = (torch.randn(Co, 3, 3, C, generator=g) * 0.05).to(torch.bfloat16)
    b = torch.randn(Co, generator=g) * 0.1
    res = torch.randn(n, H, H, Co, generator=g).to(torch.bfloat16)
    dz = torch.randn(n, H, H, Co, generator=g).to(torch.bfloat16)
    sc = torch.randn(n, H, H, C, generator=g).to(torch.bfloat16)
    ref_y = torch.relu(torch.nn.functional.conv2d(x.float().permute(0, 3, 1, 2), w.float().permute(0, 3, 1, 2), b,
                                                  padding=1).permute(0, 2, 3, 1) + res.float())
    ref_dx = torch.nn.grad.conv2d_input((n, C, H, H), w.float().permute(0, 3, 1, 2), dz.float().permute(0, 3, 1, 2),
                                        padding=1).permute(0, 2, 3, 1)
    ref_dx = (ref_dx + sc.float()) * (x.float() > 0).float()
    for name, o in outs.items():
        ey = (o["y"].float() - ref_y).norm() / ref_y.norm()
        ed = (o["dx"].float() - ref_dx).norm() / ref_dx.norm()
        assert ey < 1e-2 and ed < 1e-2, (name, float(ey), float(ed))
    for name in ("dualm", "pair"):
        assert torch.equal(outs[name]["y"], outs["generic"]["y"]), name
        assert torch.equal(outs[name]["dx"], outs["generic"]["dx"]), name


def test_dualm_short_k_projection_vs_torch():
    """1x1 / stride-2 projection (K = 64, one K-block per tile) through the dual-M kernel (ADAINF_NARROW=0 keeps
    BN = 128), against torch and bit-identical to the generic kernel (ADAINF_DUALM=0)."""
    import os, subprocess, sys
    code = f"""
import sys, torch
sys.path.insert(0, {os.path.dirname(os.path.dirname(os.path.abspath(__file__)))!r})
from paper_conf_sigcomm_shubhas23_b200 import binding as B
g = torch.Generator().manual_seed(3)
x = torch.randn(5, 30, 30, 64, generator=g).to(torch.bfloat16).cuda()
w = (torch.randn(128, 1, 1, 64, generator=g) * 0.1).to(torch.bfloat16).cuda()
b = (torch.randn(128, generator=g) * 0.1).cuda()
y = B.dbg_conv_fwd(x, w, b, 2, 0, act=0)
torch.cuda.synchronize()
torch.save(y.cpu(), sys.argv[1])
"""
    outs = {}
    for name, extra in {"generic": {"ADAINF_DUALM": "0"}, "dualm": {"ADAINF_DUALM": "1"}}.items():
        path = f"/tmp/proj_{name}.pt"
        env = dict(os.environ, ADAINF_NARROW="0", **extra)
        r = subprocess.run([sys.executable, "-c", code, path], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        outs[name] = torch.load(path)
    g = torch.Generator().manual_seed(3)
    x = torch.randn(5, 30, 30, 64, generator=g).to(torch.bfloat16)
    w = (torch.randn(128, 1, 1, 64, generator=g) * 0.1).to(torch.bfloat16)
    b = torch.randn(128, generator=g) * 0.1
    ref = torch.nn.functional.conv2d(x.float().permute(0, 3, 1, 2), w.float().permute(0, 3, 1, 2), b,
                                     stride=2).permute(0, 2, 3, 1)
    for o in outs.values():
        assert (o.float() - ref).norm() / ref.norm() < 1e-2
    assert torch.equal(outs["dualm"], outs["generic"])


@pytest.mark.parametrize("H,C,Co", [(28, 128, 256), (14, 256, 512), (9, 128, 64)])
def test_subpixel_dgrad_pair_vs_single(H, C, Co):
    """The sub-pixel stride-2 dgrad on the CTA-pair kernel (taken when 4*Cin >= 512) is bit-identical to the
    single-CTA sub-pixel GEMM (ADAINF_PAIR=0) and matches torch (+ broadcast, shortcut term, ReLU mask)."""
    import os, subprocess, sys
    code = f"""
import sys, torch
sys.path.insert(0, {os.path.dirname(os.path.dirname(os.path.abspath(__file__)))!r})
from paper_conf_sigcomm_shubhas23_b200 import binding as B
g = torch.Generator().manual_seed(3)
n = 3
Ho = ({H} + 2 - 3) // 2 + 1
w = (torch.randn({Co}, 3, 3, {C}, generator=g) * 0.05).to(torch.bfloat16).cuda()
dz = torch.randn(n, Ho, Ho, {Co}, generator=g).to(torch.bfloat16).cuda()
bc = (torch.randn(n, {C}, generator=g) * 0.01).cuda()
sc = torch.randn(n, {H}, {H}, {C}, generator=g).to(torch.bfloat16).cuda()
y = torch.randn(n, {H}, {H}, {C}, generator=g).to(torch.bfloat16).cuda()
dx = B.dbg_conv_dgrad(dz, w, {H}, {H}, 2, 1, bcast=bc, sc=sc, yact=y, mask_act=1)
torch.cuda.synchronize()
torch.save({{"dx": dx.cpu(), "w": w.cpu(), "dz": dz.cpu(), "bc": bc.cpu(), "sc": sc.cpu(), "y": y.cpu()}}, sys.argv[1])
"""
    outs = {}
    for name, pair in (("single", "0"), ("pair", "1")):
        path = f"/tmp/sp_{name}_{H}_{C}.pt"
        env = dict(os.environ, ADAINF_PAIR=pair)
        r = subprocess.run([sys.executable, "-c", code, path], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        outs[name] = torch.load(path)
    o = outs["single"]
    n = o["dz"].shape[0]
    ref = torch.nn.grad.conv2d_input((n, C, H, H), o["w"].float().permute(0, 3, 1, 2),
                                     o["dz"].float().permute(0, 3, 1, 2), stride=2, padding=1).permute(0, 2, 3, 1)
    ref = (ref + o["bc"][:, None, None, :] + o["sc"].float()) * (o["y"].float() > 0)
    for name in outs:
        assert _rel(outs[name]["dx"].float(), ref) < 8e-3, name
    assert torch.equal(outs["pair"]["dx"], outs["single"]["dx"])


@pytest.mark.parametrize("H,W", [(56, 56), (20, 20)])
def test_layer1_tile_pairs_vs_single_tiles(H, W):
    """The 64x64 window kernel's tile-pair mode (two tiles per window, B collector, ADAINF_WS_UNIT=1) is
    bit-identical to one tile per work item (ADAINF_WS_UNIT=0): forward with residual, dgrad without and with
    the shortcut term (the latter stays in single-tile mode either way)."""
    import os, subprocess, sys
    code = f"""
import sys, torch
sys.path.insert(0, {os.path.dirname(os.path.dirname(os.path.abspath(__file__)))!r})
from paper_conf_sigcomm_shubhas23_b200 import binding as B
g = torch.Generator().manual_seed(5)
n = 3
x = torch.randn(n, {H}, {W}, 64, generator=g).to(torch.bfloat16).cuda()
w = (torch.randn(64, 3, 3, 64, generator=g) * 0.05).to(torch.bfloat16).cuda()
b = (torch.randn(64, generator=g) * 0.1).cuda()
res = torch.randn(n, {H}, {W}, 64, generator=g).to(torch.bfloat16).cuda()
dz = torch.randn(n, {H}, {W}, 64, generator=g).to(torch.bfloat16).cuda()
sc = torch.randn(n, {H}, {W}, 64, generator=g).to(torch.bfloat16).cuda()
out = {{"y": B.dbg_conv_fwd(x, w, b, 1, 1, act=1, res=res).cpu(),
        "dx": B.dbg_conv_dgrad(dz, w, {H}, {W}, 1, 1, yact=x, mask_act=1).cpu(),
        "dxs": B.dbg_conv_dgrad(dz, w, {H}, {W}, 1, 1, sc=sc, yact=x, mask_act=1).cpu()}}
torch.save(out, sys.argv[1])
"""
    outs = {}
    for unit in ("0", "1"):
        path = f"/tmp/l1_{unit}_{H}_{W}.pt"
        env = dict(os.environ, ADAINF_WS_UNIT=unit)
        r = subprocess.run([sys.executable, "-c", code, path], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        outs[unit] = torch.load(path)
    for k in ("y", "dx", "dxs"):
        assert torch.equal(outs["0"][k], outs["1"][k]), k
