"""Model-level oracle pins (CPU only): parameter layout, forward vs an independent torch-fp64
interpreter, exact gradients vs torch.autograd and central finite differences, the bf16-storage
gradient vs the exact one, and SGD vs torch.optim.SGD."""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth


def mini_spec():
    """Covers conv, maxpool, projection + identity residual blocks, two exits."""
    ops = [S.conv(3, 8), S.maxpool(2, 2), S.exit_(4), S.block(16, 2), S.conv(3, 16, stride=2),
           S.conv(3, 16, residual=True), S.block(0), S.conv(3, 16), S.conv(3, 16, residual=True), S.exit_(4)]
    return {"name": "mini", "in_h": 8, "in_w": 8, "in_c": 3, "ops": ops}


def test_param_counts_match_survey():
    # tiny CNN-EE 95,188 params; ResNet-18-EE 11,181,352; detector ~5.25 M
    assert S.num_params(S.tiny_cnn_ee()) == 95188
    assert S.num_params(S.resnet18_ee()) == 11181352
    assert O.Model(S.tiny_cnn_ee()).num_params == 95188
    assert O.Model(S.resnet18_ee()).num_params == 11181352
    assert abs(S.num_params(S.tiny_yolo_det()) - 5.25e6) < 0.1e6
    # per-sample MACs: ResNet-18 full 1,813.6 M, detector 1,693.6 M
    assert abs(sum(S.macs_per_sample(S.resnet18_ee())) / 1e6 - 1813.6) < 1.0
    assert abs(sum(S.macs_per_sample(S.tiny_yolo_det())) / 1e6 - 1693.6) < 2.0


def torch_forward(spec, params, x, exact):
    """Independent fp64 interpreter built from torch.nn.functional (NCHW), bf16 rounding emulated at
    the storage points (activations, conv weights) unless exact."""
    def R(t):
        return t if exact else t.float().to(torch.bfloat16).double()

    def Fp(t):
        return t if exact else t.float().double()

    segs = {(k, i): (off, shp) for k, i, off, shp in S.param_segments(spec)}

    def seg(kind, i):
        off, shp = segs[(kind, i)]
        return params[off:off + int(np.prod(shp))].reshape(shp)

    cur = R(x.permute(0, 3, 1, 2))
    blocks, outs = [], []
    for i, o in enumerate(spec["ops"]):
        k = o["kind"]
        if k == "conv":
            w = seg("conv_w", i).permute(0, 3, 1, 2)
            w = w if exact else w.float().to(torch.bfloat16).double()
            v = Fp(Fp(F.conv2d(cur, w, stride=o["stride"], padding=o["pad"])) + seg("conv_b", i)[None, :, None, None])
            if o["residual"]:
                v = Fp(v + blocks.pop())
            if o["act"] == 1:
                v = torch.relu(v)
            elif o["act"] == 2:
                v = torch.where(v > 0, v, 0.1 * v)
            cur = R(v)
        elif k == "maxpool":
            cur = F.max_pool2d(cur, o["kh"], o["stride"], o["pad"])
        elif k == "block":
            if o["cout"] > 0:
                w = seg("proj_w", i).permute(0, 3, 1, 2)
                w = w if exact else w.float().to(torch.bfloat16).double()
                blocks.append(R(Fp(Fp(F.conv2d(cur, w, stride=o["stride"])) + seg("proj_b", i)[None, :, None, None])))
            else:
                blocks.append(cur)
        elif k == "exit":
            pooled = cur.mean(dim=(2, 3))
            outs.append(pooled @ seg("exit_w", i) + seg("exit_b", i))
    return outs


@pytest.mark.parametrize("which", ["mini", "tiny"])
def test_forward_vs_torch_interpreter(which):
    spec = mini_spec() if which == "mini" else S.tiny_cnn_ee()
    B = 6
    p = synth.init_params(spec, seed=3)
    xb, _ = synth.drifted_images(B, spec["in_h"], spec["in_w"], 3, num_classes=4, seed=1)
    x = synth.bf16_bits_to_f32(xb)
    m = O.Model(spec)
    got = m.forward(p, x)
    ref = torch_forward(spec, torch.from_numpy(p.astype(np.float64)), torch.from_numpy(x.astype(np.float64)), False)
    for k, lg in enumerate(ref):
        np.testing.assert_allclose(got["logits"][:, k, :], lg.numpy(), rtol=2e-3, atol=2e-3)
        pr = torch.softmax(lg, 1)
        np.testing.assert_allclose(got["conf"][:, k], pr.max(1).values.numpy(), rtol=1e-3, atol=1e-3)


def test_exact_grad_vs_autograd_and_fd():
    """c.1 steps 10-11: the backward derivation (CE over all exits, head grads, GAP broadcast, ReLU
    mask, first-max maxpool routing, residual copy, projection dgrad, conv dgrad/wgrad) against
    torch.autograd (fp64, exact arithmetic) and central finite differences."""
    spec = mini_spec()
    B = 5
    p = synth.init_params(spec, seed=5).astype(np.float64)
    xb, y = synth.drifted_images(B, 8, 8, 3, num_classes=4, seed=2)
    x = synth.bf16_bits_to_f32(xb)
    m = O.Model(spec)
    g = m.grad_exact(p, x, y, n_global=7)
    pt = torch.from_numpy(p.copy()).requires_grad_(True)
    outs = torch_forward(spec, pt, torch.from_numpy(x.astype(np.float64)), True)
    yt = torch.from_numpy(y.astype(np.int64))
    loss = sum(F.cross_entropy(lg, yt, reduction="sum") for lg in outs) / 7
    loss.backward()
    np.testing.assert_allclose(g, pt.grad.numpy(), rtol=1e-7, atol=1e-10)
    assert abs(m.loss(p, x, y, n_global=7) - loss.item()) < 1e-10
    rng = np.random.default_rng(0)
    h = 1e-6
    for j in rng.choice(len(p), 40, replace=False):
        pp, pm = p.copy(), p.copy()
        pp[j] += h
        pm[j] -= h
        fd = (m.loss(pp, x, y, n_global=7) - m.loss(pm, x, y, n_global=7)) / (2 * h)
        assert abs(fd - g[j]) <= 1e-6 + 1e-4 * abs(g[j]), (j, fd, g[j])


def test_bf16_grads_close_to_exact():
    """The bf16-storage gradient (what the GPU must match) stays within the 2e-2 band of the exact one
    per parameter tensor on the tiny CNN — guards against a rounding point that destroys the signal."""
    spec = S.tiny_cnn_ee()
    B = 8
    p = synth.init_params(spec, seed=7)
    xb, y = synth.drifted_images(B, 32, 32, 3, num_classes=10, seed=3)
    x = synth.bf16_bits_to_f32(xb)
    m = O.Model(spec)
    _, _, g16, _ = m.retrain_step(p, np.zeros_like(p), x, y, lr=0.0)
    ge = m.grad_exact(synth.round_bf16(p).astype(np.float64), x, y)
    for kind, _i, off, shp in S.param_segments(spec):
        n = int(np.prod(shp))
        a, b = g16[off:off + n], ge[off:off + n]
        assert np.linalg.norm(a - b) <= 5e-2 * np.linalg.norm(b) + 1e-9, kind


def test_sgd_vs_torch_optim():
    """c.1 step 12 (reading Q9): PyTorch SGD(momentum=mu, weight_decay=wd) semantics over 2 steps."""
    spec = mini_spec()
    p0 = synth.init_params(spec, seed=9)
    xb, y = synth.drifted_images(4, 8, 8, 3, num_classes=4, seed=4)
    x = synth.bf16_bits_to_f32(xb)
    m = O.Model(spec)
    lr, mu, wd = 0.05, 0.9, 1e-3
    p1, v1, g1, _ = m.retrain_step(p0, np.zeros_like(p0), x, y, lr=lr, mu=mu, wd=wd)
    p2, v2, g2, _ = m.retrain_step(p1, v1, x, y, lr=lr, mu=mu, wd=wd)
    t = torch.from_numpy(p0.copy()).requires_grad_(False)
    t = torch.nn.Parameter(t)
    opt = torch.optim.SGD([t], lr=lr, momentum=mu, weight_decay=wd)
    for g in (g1, g2):
        t.grad = torch.from_numpy(g.copy())
        opt.step()
    np.testing.assert_allclose(p2, t.detach().numpy(), rtol=1e-6, atol=1e-7)
