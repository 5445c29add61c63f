"""NEXT-3 on the GPU: ShuffleNet-EE (the paper's video-DAG classifier family) through the C-ABI — grouped 1x1
convs as one tensor-core GEMM over a block-diagonal weight, the channel shuffle folded into the producing conv's
output order, depthwise 3x3 without activation, the stride-2 unit's 3x3/2 average-pool shortcut concatenated in
front of the branch, the stride-1 unit's identity shortcut — against the oracle: a shallow well-conditioned stack at
the north_star tolerances, the full network at the oracle's own conditioning (reading Q28)."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import (bn_folded_params, check_grads, check_infer_parity, gpu_infer_single, images, oracle_sensitivity,
                    rel, to_cuda_bf16)

pytestmark = pytest.mark.gpu


def shuffle_units_spec(hw=64):
    """stem conv 3x3/2 + 3x3/2 max-pool, a stride-2 unit (avg-pool shortcut + concat, dense first 1x1) and a
    stride-1 unit (grouped 1x1, g = 8: 12 input / 4 output channels per group), an exit, another stride-2 unit
    (grouped first 1x1), the final exit (shortcuts may not span an exit, so each stage opens with a stride-2 unit)"""
    ops = [S.conv(3, 24, stride=2), S.maxpool(3, 2, 1),
           S.block(stride=2, pool=1), S.conv(1, 32), S.shuffle(8), S.conv(3, 32, stride=2, act=S.NONE, groups=32),
           S.conv(1, 72, groups=8, residual=2),
           S.block(0), S.conv(1, 32, groups=8), S.shuffle(8), S.conv(3, 32, act=S.NONE, groups=32),
           S.conv(1, 96, groups=8, residual=True), S.exit_(10),
           S.block(stride=2, pool=1), S.conv(1, 48, groups=8), S.shuffle(8),
           S.conv(3, 48, stride=2, act=S.NONE, groups=48), S.conv(1, 96, groups=8, residual=2), S.exit_(10)]
    return {"name": "shuffle_units", "in_h": hw, "in_w": hw + 4, "in_c": 3, "ops": ops}


def _params(spec, xf, seed):
    p = synth.init_params(spec, seed=seed)
    p = bn_folded_params(spec, p, xf)
    return synth.spread_exit_heads(spec, p, O.Model(spec).forward(p, xf)["logits"])


def _retrain(spec, n, seed):
    xb, y, xf = images(spec, n, seed)
    p = _params(spec, xf, seed)
    p1, _, g_o, loss_o = O.Model(spec).retrain_step(p, np.zeros_like(p), xf, y, lr=0.01, mu=0.9)
    m = B.Model(spec, n, params=p, momentum=0.9)
    st = torch.zeros(2, dtype=torch.float32, device="cuda")
    m.retrain_step(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), lr=0.01, stats=st)
    torch.cuda.synchronize()
    out = dict(p=p, p1=p1, g_o=g_o, loss_o=loss_o, g=m.get_grads(), pg=m.get_params(), loss=float(st[0].item()),
               xb=xb, y=y)
    m.close()
    return out


def test_shuffle_units_inference():
    spec = shuffle_units_spec()
    Bn = 48
    xb, _, xf = images(spec, Bn, 81)
    p = _params(spec, xf, 81)
    orc = O.Model(spec).forward(p, xf)
    taus = synth.calibrate_thresholds(orc["conf"], [0.5])
    gpu = gpu_infer_single(spec, p, xb, taus)
    nb = check_infer_parity(orc, gpu, taus)
    assert nb <= 2
    # each exit on its own, every row
    for k, t in enumerate(([0.0], [2.0])):
        g2 = gpu_infer_single(spec, p, xb, t)
        assert (g2["exit_id"] == k).all()
        for r in range(Bn):
            assert rel(g2["logits"][r], orc["logits"][r, k]) <= 2e-2, (k, r)


def test_shuffle_units_retrain_step():
    """grouped-dense wgrad gather, shuffled (row-permuted) shadow and bias, concat split + average-pool backward,
    identity shortcut: gradients 2e-2 per tensor, updated weights 1e-3, loss 2e-2"""
    spec = shuffle_units_spec()
    r = _retrain(spec, 32, 82)
    check_grads(spec, r["g"], r["g_o"])
    assert rel(r["pg"], r["p1"]) <= 1e-3
    assert rel(r["pg"] - r["p"], r["p1"] - r["p"]) <= 2e-2
    assert abs(r["loss"] - r["loss_o"]) <= 2e-2 * abs(r["loss_o"])


def test_shufflenet_ee_inference():
    spec = S.shufflenet_ee(in_hw=128)
    Bn = 12
    xb, _, xf = images(spec, Bn, 83)
    p = _params(spec, xf, 83)
    orc = O.Model(spec).forward(p, xf)
    taus = synth.calibrate_thresholds(orc["conf"], [0.3, 0.3])
    sconf, slog = oracle_sensitivity(spec, p, xb)
    band = np.maximum(1e-3, 2 * sconf[:-1])
    ltol = np.maximum(2e-2, 2 * slog)
    gpu = gpu_infer_single(spec, p, xb, taus)
    nb = check_infer_parity(orc, gpu, taus, conf_atol=max(2e-3, 2 * float(sconf.max())), band_width=band,
                            logit_tol=ltol)
    assert nb <= Bn // 2
    E = orc["conf"].shape[1]
    for k in range(E):
        t = [2.0] * (E - 1)
        if k < E - 1:
            t[k] = 0.0
        g2 = gpu_infer_single(spec, p, xb, t)
        assert (g2["exit_id"] == k).all()
        for r in range(Bn):
            assert rel(g2["logits"][r], orc["logits"][r, k]) <= ltol[k], (k, r)


def test_shufflenet_ee_retrain_step():
    """full ShuffleNet-EE g=8 at 128x128: each tensor within max(2e-2, 3x the oracle's own spread over two draws of
    20 one-ulp input flips) (reading Q28); updated weights 1e-3"""
    spec = S.shufflenet_ee(in_hw=128)
    r = _retrain(spec, 8, 84)
    m_o = O.Model(spec)
    sens = np.zeros_like(r["g_o"])
    for d in range(2):
        rng = np.random.default_rng(d)
        x2 = r["xb"].copy().view(np.uint16)
        x2.reshape(-1)[rng.choice(x2.size, 20, replace=False)] ^= 1
        _, _, g_s, _ = m_o.retrain_step(r["p"], np.zeros_like(r["p"]), synth.bf16_bits_to_f32(x2.view(r["xb"].dtype)),
                                        r["y"], lr=0.01, mu=0.9)
        sens = np.maximum(sens, np.abs(g_s - r["g_o"]))
    worst = 0.0
    for kind, i, off, shp in S.param_segments(spec):
        sl = slice(off, off + int(np.prod(shp)))
        tol = max(2e-2, 3 * float(np.linalg.norm(sens[sl]) / max(np.linalg.norm(r["g_o"][sl]), 1e-30)))
        e = rel(r["g"][sl], r["g_o"][sl])
        worst = max(worst, e / tol)
        assert e <= tol, (kind, i, e, tol)
    assert rel(r["pg"], r["p1"]) <= 1e-3
    assert abs(r["loss"] - r["loss_o"]) <= 2e-2 * abs(r["loss_o"])


@pytest.mark.parametrize("case", ["after_depthwise", "after_exit_tensor", "before_residual_conv"])
def test_shuffle_fold_rejects_unfoldable(case):
    if case == "after_depthwise":
        ops = [S.conv(3, 16), S.conv(3, 16, groups=16), S.shuffle(4), S.exit_(4)]
    elif case == "after_exit_tensor":
        ops = [S.conv(3, 16), S.conv(1, 16), S.exit_(4), S.shuffle(4), S.conv(1, 16), S.exit_(4)]
    else:
        ops = [S.conv(3, 16), S.block(0), S.conv(1, 16), S.conv(1, 16, residual=True), S.shuffle(4), S.exit_(4)]
    spec = {"name": "bad", "in_h": 16, "in_w": 16, "in_c": 3, "ops": ops}
    with pytest.raises(B.AdaInfError) as ei:
        B.Model(spec, 4)
    assert ei.value.code == B.ERR_UNSUPPORTED
