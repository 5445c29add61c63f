"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (config 2: ResNet-18-EE,
224x224, inference batch 256, retraining batch k = 1,024; config 5: a 131,072-sample selection pool, D = 512,
k = 8,192).  The oracle cannot run a 1,024-sample retraining step or a 256-sample inference batch in test time,
so the checks are (a) sampled rows the oracle computes one by one (an inference row's result does not depend on
the rest of the batch), (b) properties that hold at any size: the exit invariants (every sample exits once,
counts sum to B, nested ascending survivor lists), gradient shard additivity (the full-batch gradient equals the
sum of shard gradients scaled by 1/N_global), and the SGD closed form after one step
from zero momentum (w' = w - lr * g, P:241 / reading Q9), and (c) the full-size selection against the oracle."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import BAND, banded_rows, rel, to_cuda_bf16

pytestmark = pytest.mark.gpu

INF_B, K_SEL = 256, 1024


def test_full_size_inference_sampled_rows():
    spec = S.resnet18_ee()
    p = synth.init_params(spec, seed=1)
    protos = synth.class_prototypes(10, 224, 224, 3, seed=1244)
    xb, _ = synth.drifted_images(INF_B, 224, 224, 3, seed=100, period=1, protos=protos)
    # thresholds from the oracle on a separate 8-sample calibration batch (inputs never come from the GPU)
    cb, _ = synth.drifted_images(8, 224, 224, 3, seed=7, period=1, protos=protos)
    om = O.Model(spec)
    cal = om.forward(p, synth.bf16_bits_to_f32(cb))
    taus = [float(t) for t in synth.calibrate_thresholds(cal["conf"], [0.25, 0.25, 0.25])]
    m = B.Model(spec, INF_B, params=p)
    app = B.App([m])
    outs = B.alloc_outs(m, INF_B)
    app.infer(to_cuda_bf16(xb), taus, [outs])
    torch.cuda.synchronize()
    g = {k: v.cpu().numpy() for k, v in outs.items()}
    app.close()
    m.close()
    # invariants at full size
    E = 4
    counts = g["exit_counts"]
    assert counts.sum() == INF_B
    assert np.array_equal(np.bincount(g["exit_id"].astype(np.int64), minlength=E), counts)
    alive = np.arange(INF_B)
    for k in range(E - 1):
        n_alive = INF_B - int(counts[:k + 1].sum())
        s = g["surv_idx"][k][:n_alive]
        assert np.all(np.diff(s) > 0)
        assert set(s.tolist()) <= set(alive.tolist())
        assert set(s.tolist()) == set(np.nonzero(g["exit_id"] > k)[0].tolist())
        alive = s
    # sampled rows against the oracle, one by one
    rows = np.array([0, 37, 101, 128, 200, 255])
    orc = om.forward(p, synth.bf16_bits_to_f32(xb[rows]))
    eid, _, _ = O.exit_assign(orc["conf"], taus)
    band = banded_rows(orc["conf"], taus, eid)
    for i, r in enumerate(rows):
        if band[i]:
            continue
        assert g["exit_id"][r] == eid[i], (r, g["exit_id"][r], eid[i], orc["conf"][i])
        assert rel(g["logits"][r], orc["logits"][i, eid[i]]) <= 2e-2
    assert band.sum() <= 2


def _grads(spec, p, xb, y, idx, n_global):
    m = B.Model(spec, len(idx), params=p)
    m.retrain_step(to_cuda_bf16(np.ascontiguousarray(xb[idx])), torch.from_numpy(np.ascontiguousarray(y[idx])).cuda(),
                   n_global=n_global, lr=0.0)
    gr = m.get_grads()
    m.close()
    return gr


def test_full_size_retrain_shard_additivity_and_sgd_closed_form():
    spec = S.resnet18_ee()
    p = synth.init_params(spec, seed=1)
    protos = synth.class_prototypes(10, 224, 224, 3, seed=1244)
    xb, y = synth.drifted_images(K_SEL, 224, 224, 3, seed=101, period=0, protos=protos)
    full = _grads(spec, p, xb, y, np.arange(K_SEL), K_SEL)
    assert np.isfinite(full).all()
    parts = sum(_grads(spec, p, xb, y, np.arange(K_SEL)[r::4], K_SEL) for r in range(4))
    worst = 0.0
    for kind, i, off, shp in S.param_segments(spec):
        n = int(np.prod(shp))
        r = rel(parts[off:off + n], full[off:off + n])
        worst = max(worst, r)
        assert r <= 1e-3, (kind, i, r)
    # one SGD step from zero momentum: w' = w - lr * g exactly (fp32, no FMA), momentum then = g
    lr = np.float32(0.01)
    m = B.Model(spec, K_SEL, params=p, momentum=0.9)
    m.retrain_step(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), n_global=K_SEL, lr=float(lr))
    w1 = m.get_params()
    m.close()
    expect = (p.astype(np.float32) - lr * full.astype(np.float32)).astype(np.float32)
    assert rel(w1, expect) <= 1e-6
    assert rel(w1 - p, expect - p) <= 2e-2


@pytest.mark.parametrize("N,D,P,M,k", [(131072, 512, 64, 1, 8192), (32768, 512, 64, 256, 2048)])
def test_full_size_selection(N, D, P, M, k):
    """Config 5 pool (heavy drift): 131,072 candidates, D = 512 -> P = 64, k = 8,192 (and an M = 256 reference
    variant) against the oracle: eligible count, exact index set outside the band, ascending output."""
    Xb, Wb, ref = synth.embeddings(N, D, P, seed=5, M=M)
    ex = (np.random.default_rng(5).random(N) < 0.1).astype(np.uint8)
    X = torch.from_numpy(Xb.view(np.int16)).cuda().view(torch.bfloat16).reshape(N, D)
    W = torch.from_numpy(Wb.view(np.int16)).cuda().view(torch.bfloat16).reshape(D, P)
    idx, dd, cnt = B.select_retrain(X, W, torch.from_numpy(ref).cuda(), k, exclude=torch.from_numpy(ex).cuda())
    torch.cuda.synchronize()
    cnt = int(cnt.item())
    idx = idx.cpu().numpy()[:cnt]
    oi, od, oc, odist = O.select(synth.bf16_bits_to_f32(Xb).reshape(N, D), synth.bf16_bits_to_f32(Wb).reshape(D, P),
                                 ref, k, exclude=ex)
    assert cnt == oc == k
    assert np.all(np.diff(idx) > 0) and not ex[idx].any()
    el = ex == 0
    dk = np.sort(odist[el])[::-1][k - 1]
    banded = np.abs(odist - dk) < BAND
    assert set(i for i in idx.tolist() if not banded[i]) == set(i for i in oi.tolist() if not banded[i])
