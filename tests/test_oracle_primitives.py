"""Pins of the oracle's primitives against things other than itself (CPU only).

Each test names the passage / reading it pins and what a plausible bug would break.
"""
import math

import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import synth


def test_bf16_rne_matches_torch():
    # hand-picked ties (exactly half-way) plus random values: torch's bf16 cast is RNE
    ties = np.array([1.0 + 2 ** -8, 1.0 + 3 * 2 ** -8, -(1.0 + 2 ** -8), 2 ** -130, 3.0e38], np.float32)
    rnd = np.random.default_rng(0).standard_normal(10000).astype(np.float32) * 10
    for x in (ties, rnd):
        ref = torch.from_numpy(x).to(torch.bfloat16).to(torch.float32).numpy()
        np.testing.assert_array_equal(O.bf16(x), ref)
        np.testing.assert_array_equal(synth.round_bf16(x), ref)


def _torch_conv(x, w, s, p):
    xt = torch.from_numpy(x.astype(np.float64)).permute(2, 0, 1)[None]
    wt = torch.from_numpy(w.astype(np.float64)).permute(0, 3, 1, 2)
    return torch.nn.functional.conv2d(xt, wt, stride=s, padding=p)[0].permute(1, 2, 0).numpy()


@pytest.mark.parametrize("H,W,C,Co,K,s,p", [(7, 5, 3, 4, 3, 1, 1), (9, 9, 8, 6, 3, 2, 1), (11, 10, 3, 5, 7, 2, 3),
                                            (6, 6, 16, 8, 1, 2, 0), (5, 5, 4, 3, 2, 2, 0)])
def test_conv_acc_vs_torch_fp64(H, W, C, Co, K, s, p):
    """c.1 step 2 conv definition; library special case torch conv2d fp64 on bf16-rounded operands.
    A transposed weight (kh<->kw) or a wrong padding sign fails here (non-square kernels/inputs)."""
    rng = np.random.default_rng(H * 100 + K)
    x = O.bf16(rng.standard_normal((H, W, C)).astype(np.float32))
    w = O.bf16(rng.standard_normal((Co, K, K, C)).astype(np.float32))
    got = O.conv_acc(x, w, s, p)
    ref = _torch_conv(x, w, s, p)
    assert got.shape == ref.shape
    np.testing.assert_allclose(got, ref.astype(np.float32), rtol=1e-6, atol=1e-6)


def test_conv_acc_closed_forms():
    rng = np.random.default_rng(3)
    x = O.bf16(rng.standard_normal((6, 7, 5)).astype(np.float32))
    # identity 1x1 kernel -> copy of the input
    w = np.zeros((5, 1, 1, 5), np.float32)
    for c in range(5):
        w[c, 0, 0, c] = 1
    np.testing.assert_array_equal(O.conv_acc(x, w, 1, 0), x)
    # all-ones 3x3 kernel on a constant-1 single channel -> box counts (9 inside, 6 edges, 4 corners)
    ones = np.ones((4, 4, 1), np.float32)
    got = O.conv_acc(ones, np.ones((1, 3, 3, 1), np.float32), 1, 1)[..., 0]
    ref = np.array([[4, 6, 6, 4], [6, 9, 9, 6], [6, 9, 9, 6], [4, 6, 6, 4]], np.float32)
    np.testing.assert_array_equal(got, ref)
    # zero input -> zero accumulator
    assert not O.conv_acc(np.zeros((5, 5, 3), np.float32), rng.standard_normal((2, 3, 3, 3)), 1, 1).any()


def test_maxpool_vs_torch():
    rng = np.random.default_rng(5)
    x = O.bf16(rng.standard_normal((9, 8, 6)).astype(np.float32))
    for k, s, p in ((2, 2, 0), (3, 2, 1), (3, 1, 1)):
        got = O.maxpool(x, k, s, p)
        ref = torch.nn.functional.max_pool2d(torch.from_numpy(x).permute(2, 0, 1)[None], k, s, p)[0]
        np.testing.assert_array_equal(got, ref.permute(1, 2, 0).numpy())


def test_softmax_stats_closed_forms():
    """Q1/Q7: conf = max softmax, natural-log entropy, lowest-index argmax (Q6)."""
    for C in (2, 4, 10):
        conf, ent, pred = O.softmax_stats(np.full(C, 0.37, np.float32))
        assert abs(conf - 1.0 / C) < 1e-7 and abs(ent - math.log(C)) < 1e-6 and pred == 0
    l = np.zeros(10, np.float32)
    l[3] = 40.0
    conf, ent, pred = O.softmax_stats(l)
    assert pred == 3 and abs(conf - (1 - 9 * math.exp(-40))) < 1e-7 and ent < 1e-12
    for d in (-3.0, 0.5, 2.0):
        conf, ent, pred = O.softmax_stats(np.array([0.0, d], np.float32))
        sig = 1 / (1 + math.exp(-abs(d)))
        assert abs(conf - sig) < 1e-7
        assert abs(ent - (-(sig * math.log(sig) + (1 - sig) * math.log(1 - sig)))) < 1e-6
        assert pred == (1 if d > 0 else 0)
    # tie between the top two -> the lower index
    assert O.softmax_stats(np.array([0.1, 0.9, 0.9, 0.2], np.float32))[2] == 1


def test_exit_head_vs_torch():
    rng = np.random.default_rng(7)
    f = O.bf16(rng.standard_normal((5, 6, 12)).astype(np.float32))
    Wk = rng.standard_normal((12, 7)).astype(np.float32)
    bk = rng.standard_normal(7).astype(np.float32)
    pooled, logits, conf, ent, pred = O.exit_head(f, Wk, bk)
    ft = torch.from_numpy(f.astype(np.float64))
    pr = ft.mean(dim=(0, 1))
    lr = pr @ torch.from_numpy(Wk.astype(np.float64)) + torch.from_numpy(bk.astype(np.float64))
    p = torch.softmax(lr, 0)
    np.testing.assert_allclose(pooled, pr.numpy(), rtol=1e-6, atol=1e-7)
    np.testing.assert_allclose(logits, lr.numpy(), rtol=1e-5, atol=1e-5)
    assert abs(conf - p.max().item()) < 1e-6
    assert abs(ent - float(-(p * p.log()).sum())) < 1e-5
    assert pred == int(torch.argmax(lr))


def test_exit_assign_invariants_and_special_cases():
    """P:96/P:229 exit rule + c.1 step 5 compaction: invariants every sample exits once, counts sum to
    B, survivors ascending and nested; tau=0 -> all at exit 0; tau>1 -> all at the final exit;
    raising tau_k only moves samples from exit k to later exits."""
    rng = np.random.default_rng(11)
    B, E = 257, 4
    conf = rng.random((B, E)).astype(np.float32)
    tau = np.array([0.8, 0.6, 0.5], np.float32)
    eid, surv, counts = O.exit_assign(conf, tau)
    assert counts.sum() == B
    np.testing.assert_array_equal(np.bincount(eid, minlength=E), counts)
    prev = set(range(B))
    for k in range(E - 1):
        s = surv[k][surv[k] >= 0]
        assert np.all(np.diff(s) > 0)
        assert set(s.tolist()) <= prev
        assert len(s) == B - counts[:k + 1].sum()
        prev = set(s.tolist())
    # brute force of the rule itself
    for n in range(B):
        first = next((k for k in range(E - 1) if conf[n, k] >= tau[k]), E - 1)
        assert eid[n] == first
    assert (O.exit_assign(conf, np.zeros(E - 1, np.float32))[0] == 0).all()
    assert (O.exit_assign(conf, np.full(E - 1, 1.5, np.float32))[0] == E - 1).all()
    tau2 = tau.copy()
    tau2[1] = 0.9
    eid2 = O.exit_assign(conf, tau2)[0]
    changed = eid2 != eid
    assert np.all(eid[changed] == 1) and np.all(eid2[changed] > 1)


def test_detect_closed_forms():
    """Q18 decode: t=0 -> box centred at (col+0.5)*stride with the anchor size; score = sigmoid(obj) *
    sigmoid(cls*); clamping to the image; ascending linear-index order; threshold on score."""
    G, A, NC, stride = 3, 2, 2, 32
    aw = [20.0, 30.0, 200.0, 100.0]
    raw = np.zeros((2, G, G, A * (5 + NC)), np.float32)
    raw[..., 4] = -10  # anchor 0 objectness off
    raw[..., 5 + NC + 4] = -10
    raw[1, 2, 1, 4] = 3.0          # frame 1, row 2, col 1, anchor 0: obj on
    raw[1, 2, 1, 5 + 1] = 2.0      # class 1 wins
    raw[0, 0, 0, 5 + NC + 4] = 5.0  # frame 0, cell 0, anchor 1: big anchor -> clamped
    det, n = O.detect(raw, A, NC, aw, stride, 96, 96, tau_det=0.3)
    assert n == 2
    # ascending linear index: frame 0 first
    f0 = det[0]
    assert f0[0] == 0 and f0[1] == 0 and f0[2] == 1 and f0[3] == 0
    s = 1 / (1 + math.exp(-5.0)) * 0.5
    assert abs(f0[4] - s) < 1e-6
    # centre (0.5*32, 0.5*32) = 16, w=200,h=100 -> clamped to [0, 96]
    np.testing.assert_allclose(f0[5:], [0, 0, 96, 66], atol=1e-4)
    f1 = det[1]
    assert f1[0] == 1 and f1[1] == 2 * G + 1 and f1[2] == 0 and f1[3] == 1
    cx, cy = 1.5 * 32, 2.5 * 32
    np.testing.assert_allclose(f1[5:], [cx - 10, cy - 15, cx + 10, min(cy + 15, 96)], atol=1e-4)
    assert abs(f1[4] - (1 / (1 + math.exp(-3))) * (1 / (1 + math.exp(-2)))) < 1e-6
    # raising tau above both scores -> none
    assert O.detect(raw, A, NC, aw, stride, 96, 96, tau_det=0.99)[1] == 0


def test_detect_multi_two_scales_brute_force():
    """Two-scale decode (NEXT-3, reading Q18c) against a plain per-candidate loop written from the definition: each
    head's own stride and anchors, the cell index re-based past the earlier heads' cells, rows in ascending
    (frame, head, cell, anchor) order; a swapped stride or anchor set, or a missing re-base, fails here."""
    rng = np.random.default_rng(7)
    A, NC, B = 2, 3, 3
    heads = [(3, 32, [30.0, 40.0, 90.0, 70.0]), (6, 16, [8.0, 10.0, 14.0, 20.0])]
    raws = [rng.normal(0, 1.5, (B, G, G, A * (5 + NC))).astype(np.float32) for G, _, _ in heads]
    img = 96
    sig = lambda v: 1.0 / (1.0 + math.exp(-float(v)))
    exp_rows, scores = [], []
    for f in range(B):
        off = 0
        for (G, st, aw), raw in zip(heads, raws):
            for r in range(G):
                for c in range(G):
                    for a in range(A):
                        v = raw[f, r, c, a * (5 + NC):(a + 1) * (5 + NC)]
                        cs = int(np.argmax(v[5:]))
                        sc = sig(v[4]) * sig(v[5 + cs])
                        scores.append(sc)
                        cx, cy = (c + sig(v[0])) * st, (r + sig(v[1])) * st
                        w, h = aw[2 * a] * math.exp(min(v[2], 4.0)), aw[2 * a + 1] * math.exp(min(v[3], 4.0))
                        box = [min(max(cx - w / 2, 0), img), min(max(cy - h / 2, 0), img),
                               min(max(cx + w / 2, 0), img), min(max(cy + h / 2, 0), img)]
                        exp_rows.append((f, off + r * G + c, a, cs, sc, *box))
            off += G * G
    s_sorted = np.sort(scores)
    lo, hi = int(0.6 * len(s_sorted)), int(0.9 * len(s_sorted))  # widest gap between the 60th and 90th percentile
    gi = np.argmax(np.diff(s_sorted[lo:hi])) + lo
    tau = float(0.5 * (s_sorted[gi] + s_sorted[gi + 1]))
    want = [r for r in exp_rows if r[4] >= tau]
    det, n = O.detect_multi(raws, A, NC, [h[2] for h in heads], [h[1] for h in heads], img, img, tau)
    assert n == len(want) == det.shape[0] > 3
    for got, w in zip(det, want):
        assert tuple(int(v) for v in got[:4]) == w[:4]
        np.testing.assert_allclose(got[4:], w[4:], rtol=1e-5, atol=1e-3)


def test_crop_identity_constant_and_grid_sample():
    rng = np.random.default_rng(2)
    H, W, Cc = 12, 10, 3
    fr = O.bf16(rng.standard_normal((H, W, Cc)).astype(np.float32))
    # identity: full-image box at the image's own size -> exact copy
    np.testing.assert_array_equal(O.crop(fr, (0, 0, W, H), H, W), fr)
    # constant image -> constant crop
    const = np.full((H, W, Cc), np.float32(0.75))
    assert (O.crop(const, (1.3, 2.2, 7.9, 9.1), 5, 6) == np.float32(0.75)).all()
    # library special case: grid_sample(bilinear, align_corners=False, border) on the same sample points
    box = (1.5, 0.75, 8.25, 11.0)
    ch, cw = 7, 9
    got = O.crop(fr, box, ch, cw)
    x0, y0, x1, y1 = box
    xs = x0 + (np.arange(cw) + 0.5) * (x1 - x0) / cw - 0.5
    ys = y0 + (np.arange(ch) + 0.5) * (y1 - y0) / ch - 0.5
    gx = (xs + 0.5) / W * 2 - 1
    gy = (ys + 0.5) / H * 2 - 1
    grid = torch.from_numpy(np.stack(np.meshgrid(gx, gy), -1)[None].astype(np.float64))
    ref = torch.nn.functional.grid_sample(torch.from_numpy(fr.astype(np.float64)).permute(2, 0, 1)[None], grid,
                                          mode="bilinear", padding_mode="border", align_corners=False)
    ref = ref[0].permute(1, 2, 0).numpy()
    np.testing.assert_allclose(got, ref, rtol=1e-2, atol=1e-2)  # bf16 output rounding


def test_select_closed_forms_and_bruteforce():
    """P:195 cosine distance to the old mean after projection; Q15 ties -> lower index, ascending output;
    P:243 excluded samples never selected; Q17 zero vector -> d = 1."""
    D = 4
    mu = np.array([[1.0, 0, 0, 0]], np.float32)
    X = np.array([[2, 0, 0, 0], [0, 3, 0, 0], [-1, 0, 0, 0], [0, 0, 0, 0], [1, 1, 0, 0]], np.float32)
    idx, dd, cnt, dist = O.select(X, None, mu, 5)
    np.testing.assert_allclose(dist, [0, 1, 2, 1, 1 - 1 / math.sqrt(2)], atol=1e-6)
    assert cnt == 5 and list(idx) == [0, 1, 2, 3, 4]
    idx, dd, cnt, _ = O.select(X, None, mu, 2)
    assert list(idx) == [1, 2]  # d=2 (idx 2) and the lower of the two d=1 ties (idx 1)
    ex = np.array([0, 1, 0, 0, 0], np.uint8)
    idx, _, cnt, _ = O.select(X, None, mu, 2, exclude=ex)
    assert list(idx) == [2, 3]
    idx, _, cnt, _ = O.select(X, None, mu, 10, exclude=ex)
    assert cnt == 4 and 1 not in idx
    # brute force with a projection and M>1 references
    rng = np.random.default_rng(4)
    N, D, P, M = 300, 16, 5, 3
    X = O.bf16(rng.standard_normal((N, D)).astype(np.float32))
    Wp = O.bf16(rng.standard_normal((D, P)).astype(np.float32))
    ref = rng.standard_normal((M, D)).astype(np.float32)
    idx, dd, cnt, dist = O.select(X, Wp, ref, 37)
    Y = X.astype(np.float64) @ Wp.astype(np.float64)
    R = ref.astype(np.float64) @ Wp.astype(np.float64)
    cos = (Y @ R.T) / np.maximum(np.linalg.norm(Y, axis=1)[:, None] * np.linalg.norm(R, axis=1)[None], 1e-12)
    d = (1 - cos).min(1)
    np.testing.assert_allclose(dist, d, rtol=1e-5, atol=1e-6)
    order = sorted(range(N), key=lambda i: (-np.float32(d[i]), i))[:37]
    assert list(idx) == sorted(order)


def test_iou_closed_forms():
    """NEXT-3 NMS (reading Q18b): IoU = inter / (area_a + area_b - inter) in fp32."""
    assert abs(O.iou([0, 0, 2, 2], [1, 1, 3, 3]) - 1.0 / 7.0) < 1e-7
    assert O.iou([1, 2, 5, 7], [1, 2, 5, 7]) == 1.0
    assert O.iou([0, 0, 1, 1], [2, 2, 3, 3]) == 0.0
    assert O.iou([0, 0, 1, 1], [1, 0, 2, 1]) == 0.0  # touching edges: zero intersection
    assert abs(O.iou([0, 0, 4, 4], [1, 1, 3, 3]) - 0.25) < 1e-7  # contained
    assert O.iou([0, 0, 0, 0], [0, 0, 0, 0]) == 0.0  # zero-area union


def _det_rows(rows):
    return np.array([[f, i, 0, c, s, x0, y0, x1, y1] for i, (f, c, s, x0, y0, x1, y1) in enumerate(rows)],
                    np.float32)


def test_nms_closed_forms_and_greedy_chain():
    thr = 0.45
    # identical boxes, same frame and class: the higher score survives; equal scores -> the lower row survives
    k, n = O.nms(_det_rows([(0, 0, 0.9, 0, 0, 10, 10), (0, 0, 0.8, 0, 0, 10, 10)]), thr)
    assert k.tolist() == [1, 0] and n == 1
    k, _ = O.nms(_det_rows([(0, 0, 0.8, 0, 0, 10, 10), (0, 0, 0.9, 0, 0, 10, 10)]), thr)
    assert k.tolist() == [0, 1]
    k, _ = O.nms(_det_rows([(0, 0, 0.7, 0, 0, 10, 10), (0, 0, 0.7, 0, 0, 10, 10)]), thr)
    assert k.tolist() == [1, 0]
    # other class or other frame never suppresses
    assert O.nms(_det_rows([(0, 0, 0.9, 0, 0, 10, 10), (0, 1, 0.8, 0, 0, 10, 10)]), thr)[0].tolist() == [1, 1]
    assert O.nms(_det_rows([(0, 0, 0.9, 0, 0, 10, 10), (1, 0, 0.8, 0, 0, 10, 10)]), thr)[0].tolist() == [1, 1]
    # IoU exactly at the threshold is kept (suppression is strict >): [0,0,2,2] vs [1,1,3,3] -> 1/7
    t7 = np.float32(1.0) / np.float32(7.0)
    assert O.nms(_det_rows([(0, 0, 0.9, 0, 0, 2, 2), (0, 0, 0.8, 1, 1, 3, 3)]), float(t7))[0].tolist() == [1, 1]
    assert O.nms(_det_rows([(0, 0, 0.9, 0, 0, 2, 2), (0, 0, 0.8, 1, 1, 3, 3)]), float(t7) * 0.99)[0].tolist() == [1, 0]
    # greedy chain: A suppresses B, B (not kept) cannot suppress C although IoU(B, C) > thr
    rows = [(0, 0, 0.9, 0, 0, 10, 10), (0, 0, 0.8, 3, 0, 13, 10), (0, 0, 0.7, 6, 0, 16, 10)]
    d = _det_rows(rows)
    assert O.iou(d[0, 5:], d[1, 5:]) > thr and O.iou(d[1, 5:], d[2, 5:]) > thr and O.iou(d[0, 5:], d[2, 5:]) < thr
    assert O.nms(d, thr)[0].tolist() == [1, 0, 1]


def _iou_np(a, b):
    f = np.float32
    iw = max(f(0), min(a[2], b[2]) - max(a[0], b[0]))
    ih = max(f(0), min(a[3], b[3]) - max(a[1], b[1]))
    inter = f(iw * ih)
    uni = f(f(f((a[2] - a[0]) * (a[3] - a[1])) + f((b[2] - b[0]) * (b[3] - b[1]))) - inter)
    return f(inter / uni) if uni > 0 else f(0)


def test_nms_textbook_loop_and_invariants():
    """Against the textbook loop (repeatedly take the best remaining box of a (frame, class) group, drop every
    box overlapping it by more than the threshold) and the two invariants of greedy NMS: kept boxes of a group
    overlap pairwise by <= thr, and every dropped box overlaps a kept box that precedes it in score order."""
    rng = np.random.default_rng(3)
    thr = 0.45
    for trial in range(20):
        n = int(rng.integers(1, 60))
        x0 = rng.uniform(0, 80, n)
        y0 = rng.uniform(0, 80, n)
        w = rng.uniform(2, 30, n)
        h = rng.uniform(2, 30, n)
        sc = np.round(rng.uniform(0.1, 1.0, n), 2)  # rounded: ties occur
        rows = [(int(rng.integers(0, 2)), int(rng.integers(0, 3)), sc[i], x0[i], y0[i], x0[i] + w[i], y0[i] + h[i])
                for i in range(n)]
        d = _det_rows(rows)
        keep, _ = O.nms(d, thr)
        ref = np.zeros(n, np.uint8)
        for f_ in (0, 1):
            for c_ in range(3):
                rem = [i for i in range(n) if d[i, 0] == f_ and d[i, 3] == c_]
                while rem:
                    best = min(rem, key=lambda i: (-d[i, 4], i))
                    ref[best] = 1
                    rem = [i for i in rem if i != best and not _iou_np(d[best, 5:], d[i, 5:]) > np.float32(thr)]
        assert keep.tolist() == ref.tolist(), trial
        for i in range(n):
            same = [j for j in range(n) if j != i and d[j, 0] == d[i, 0] and d[j, 3] == d[i, 3]]
            if keep[i]:
                assert all(not (keep[j] and _iou_np(d[i, 5:], d[j, 5:]) > np.float32(thr)) for j in same)
            else:
                assert any(keep[j] and (d[j, 4], -j) > (d[i, 4], -i) and _iou_np(d[i, 5:], d[j, 5:]) > np.float32(thr)
                           for j in same)
