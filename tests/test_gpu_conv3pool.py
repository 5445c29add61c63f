"""conv3pool.cu: 3x3/1 conv + bias + act + 2x2/2 max-pool in one tensor-core kernel (the C3 detector's few-channel
layers, reading Q18) against torch (fp64 conv of the same bf16 operands, bias and act in fp32, bf16 rounding, then the
pool — the oracle's storage points), at widths spanning one and two 128-column tiles with ragged tails, the row-pair
and the space-to-depth first-layer modes, and leaky-ReLU / none / ReLU."""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

from paper_conf_sigcomm_shubhas23_b200 import binding as B

pytestmark = pytest.mark.gpu


def ref(x, w, b, act):
    z = F.conv2d(x.double().permute(0, 3, 1, 2), w.double().permute(0, 3, 1, 2), padding=1).float()
    z = z + b[None, :, None, None]
    if act == 1:
        z = torch.relu(z)
    elif act == 2:
        z = torch.where(z > 0, z, z * torch.tensor(0.1, dtype=torch.float32))
    z = z.to(torch.bfloat16).float()
    return F.max_pool2d(z, 2, 2).permute(0, 2, 3, 1).contiguous()


@pytest.mark.parametrize("n,H,W,C,Co,act,first", [
    (3, 20, 300, 16, 32, 2, False),    # two column tiles, ragged (300 = 256 + 44)
    (2, 24, 104, 32, 64, 2, False),    # one tile, 104 of 128 columns
    (2, 10, 130, 16, 128, 1, False),   # 130 = 128 + 2 (one column of the second tile pair)
    (2, 8, 64, 32, 96, 0, False),
    (2, 16, 416, 4, 16, 2, True),      # the detector's first layer geometry (s2d grid 8 x 208: two tiles)
    (3, 12, 40, 4, 32, 1, True),
])
def test_conv3_pool_vs_torch(n, H, W, C, Co, act, first):
    g = torch.Generator(device="cpu").manual_seed(H * 7 + W)
    cin_real = 3 if first else C
    x = torch.randn(n, H, W, C, generator=g)
    if first:
        x[..., cin_real:] = 0
    x = x.to(torch.bfloat16)
    w = (torch.randn(Co, 3, 3, C, generator=g) * (1.0 / np.sqrt(9 * cin_real))).to(torch.bfloat16)
    if first:
        w[..., cin_real:] = 0
    b = torch.randn(Co, generator=g) * 0.1
    y = B.dbg_conv3_pool(x.cuda(), w.cuda(), b.cuda(), act=act, first=first, cin_real=cin_real)
    torch.cuda.synchronize()
    r = ref(x.float(), w.float(), b, act)
    yg = y.float().cpu()
    # fp32 tensor-core accumulation vs fp64: a rare bf16 rounding flip of a pre-pool value (1 ulp = 2^-8 relative)
    d = (yg - r).abs()
    tol = 2.0 ** -7 * r.abs().clamp_min(2.0 ** -6)
    assert (d <= tol).all(), (d.max().item(), (d > tol).sum().item())
    assert (d > 0).float().mean().item() < 5e-3


def test_conv3_pool_rejects_other_geometry():
    x = torch.zeros(1, 8, 8, 64, dtype=torch.bfloat16, device="cuda")
    w = torch.zeros(32, 3, 3, 64, dtype=torch.bfloat16, device="cuda")
    b = torch.zeros(32, device="cuda")
    with pytest.raises(B.AdaInfError) as ei:
        B.dbg_conv3_pool(x, w, b)
    assert ei.value.code == B.ERR_SHAPE
