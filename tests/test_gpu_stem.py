"""Space-to-depth ResNet stem (7x7/2 conv + bias + ReLU + 3x3/2 max-pool, csrc/stem.cu) against torch fp32 on the
same bf16 operands, through the debug C-ABI (include/adainf_debug.h).  The forward compares pooled values and
first-argmax indices; the weight gradient compares dW and the fused bias gradient."""
import pytest
import torch

from paper_conf_sigcomm_shubhas23_b200 import binding as B

pytestmark = pytest.mark.gpu


def _rel(a, b):
    a, b = a.double(), b.double()
    return float((a - b).norm() / b.norm().clamp_min(1e-30))


def _ref_stem(x, w, b):
    """conv -> bias -> ReLU -> bf16, then 3x3/2 pad-1 max-pool with the FIRST maximum in row-major window order."""
    y = torch.nn.functional.conv2d(x.float().permute(0, 3, 1, 2), w.float().permute(0, 3, 1, 2), b, stride=2, padding=3)
    y = torch.relu(y).to(torch.bfloat16).float()
    n, C, H, W = y.shape
    yp = torch.nn.functional.pad(y, (1, 1, 1, 1), value=float("-inf"))
    cols = torch.nn.functional.unfold(yp, 3, stride=2)  # [n, C*9, L]
    cols = cols.view(n, C, 9, -1)
    best, arg = cols.max(dim=2)
    Hp, Wp = (H - 1) // 2 + 1, (W - 1) // 2 + 1
    best = best.view(n, C, Hp, Wp).permute(0, 2, 3, 1)
    arg = arg.view(n, C, Hp, Wp).permute(0, 2, 3, 1)
    # torch.max over dim returns an index of a maximal value; make it the first one explicitly
    first = (cols == cols.max(dim=2, keepdim=True).values).float().argmax(dim=2)
    first = first.view(n, C, Hp, Wp).permute(0, 2, 3, 1)
    return best, first, y


CASES = [(2, 224, 224, 3), (3, 64, 48, 3), (2, 30, 34, 1), (5, 16, 16, 4), (1, 250, 90, 3)]


@pytest.mark.parametrize("case", CASES)
def test_stem_fwd(case):
    n, H, W, cin = case
    g = torch.Generator().manual_seed(3)
    x = torch.randn(n, H, W, cin, generator=g).to(torch.bfloat16).cuda()
    w = (torch.randn(64, 7, 7, cin, generator=g) * (1.0 / (49 * cin)) ** 0.5).to(torch.bfloat16).cuda()
    b = (torch.randn(64, generator=g) * 0.1).cuda()
    pooled, am = B.dbg_stem_fwd(x, w, b)
    torch.cuda.synchronize()
    ref, ref_arg, _ = _ref_stem(x, w, b)
    assert pooled.shape == ref.shape
    assert _rel(pooled.float(), ref) < 5e-3
    # pooled values are bf16 of the same rounding except where fp32 summation order flips a rounding
    assert (pooled.float() == ref).float().mean() > 0.98
    # a window whose max is 0 (every ReLU output <= 0) carries the masked code 255 (no gradient routed)
    ref_arg = torch.where(ref == 0, torch.full_like(ref_arg, 255), ref_arg)
    assert (am.long() == ref_arg).float().mean() > 0.98
    assert torch.all((am == 255) == (pooled.float() == 0))


def test_stem_fwd_all_negative_window_and_ties():
    """Windows where every ReLU output is 0: the pooled value is 0 and the code is 255 (ReLU' = 0 folded in:
    no gradient is routed through such a window)."""
    n, H, W, cin = 2, 32, 32, 3
    x = torch.zeros(n, H, W, cin, dtype=torch.bfloat16).cuda()
    w = torch.zeros(64, 7, 7, cin, dtype=torch.bfloat16).cuda()
    b = torch.full((64,), -1.0).cuda()
    pooled, am = B.dbg_stem_fwd(x, w, b)
    torch.cuda.synchronize()
    assert torch.all(pooled.float() == 0)
    assert torch.all(am == 255)


@pytest.mark.parametrize("case", CASES)
def test_stem_wgrad(case):
    n, H, W, cin = case
    g = torch.Generator().manual_seed(4)
    x = torch.randn(n, H, W, cin, generator=g).to(torch.bfloat16).cuda()
    dz = torch.randn(n, H // 2, W // 2, 64, generator=g).to(torch.bfloat16).cuda()
    # sparse like a max-pool gradient: ~3/4 zeros
    dz = dz * (torch.rand(n, H // 2, W // 2, 64, generator=g) < 0.25).to(torch.bfloat16).cuda()
    dw, db = B.dbg_stem_wgrad(x, dz)
    torch.cuda.synchronize()
    ref = torch.nn.grad.conv2d_weight(x.float().permute(0, 3, 1, 2), (64, cin, 7, 7), dz.float().permute(0, 3, 1, 2),
                                      stride=2, padding=3).permute(0, 2, 3, 1)
    assert _rel(dw, ref) < 1e-4
    assert _rel(db, dz.float().sum(dim=(0, 1, 2))) < 1e-5
    dw2, db2 = B.dbg_stem_wgrad(x, dz)
    torch.cuda.synchronize()
    diff = (dw2 - dw).abs()
    assert torch.equal(dw, dw2), ("dw", float(diff.max()), torch.nonzero(diff)[:8].tolist())
    assert torch.equal(db, db2), ("db", float((db2 - db).abs().max()))
