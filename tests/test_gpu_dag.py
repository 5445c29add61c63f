"""Application-DAG parity (Fig. 1): detector -> on-device decode / routing /
crop -> vehicle + person classifiers, and whole-input routing by predicted class (audio DAG, Q24).

Contract (SURVEY c.3 Q20): detections (frame, cell, anchor, class), routing destinations and order are
bit-exact outside the tau_det band; boxes within 0.5 px + 1e-3 * size; crops and downstream outputs are
checked stage-isolated (the oracle re-crops from the GPU's det_table boxes)."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import BAND, rel, to_cuda_bf16

pytestmark = pytest.mark.gpu


def small_cls(num_classes, hw=32, in_c=3):
    return {"name": "cls", "in_h": hw, "in_w": hw, "in_c": in_c,
            "ops": [S.conv(3, 32), S.maxpool(2, 2), S.conv(3, 64), S.maxpool(2, 2), S.exit_(num_classes),
                    S.conv(3, 64), S.exit_(num_classes)]}


def _calib_tau(scores, frac):
    s = np.sort(scores)[::-1]
    k = int(frac * len(s))
    best, bi = -1, k
    for j in range(max(1, k - 20), min(len(s) - 1, k + 20)):
        if s[j - 1] - s[j] > best:
            best, bi = s[j - 1] - s[j], j
    return float(0.5 * (s[bi - 1] + s[bi]))


def test_video_dag_detector_routing_crops():
    Bn, hw, crop = 6, 96, 32
    det_spec = S.tiny_yolo_det(in_hw=hw)
    A, NC = 3, 2
    p_det = synth.det_head_params(det_spec, synth.init_params(det_spec, seed=21), obj_bias=0.0)
    veh, per = small_cls(10), small_cls(8)
    p_veh, p_per = synth.init_params(veh, seed=22), synth.init_params(per, seed=23)
    xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=21)
    xf = synth.bf16_bits_to_f32(xb)
    # oracle detector raw output and scores -> tau_det in a wide gap (~1/3 of candidates detected)
    orc_raw = O.Model(det_spec).forward(p_det, xf, want_det=True)["det"]
    G = orc_raw.shape[1]
    aw = S.YOLO_ANCHORS
    sig = lambda v: 1 / (1 + np.exp(-v.astype(np.float64)))
    r5 = orc_raw.reshape(Bn, G, G, A, 5 + NC)
    scores = (sig(r5[..., 4]) * sig(r5[..., 5:].max(-1))).reshape(-1)
    tau_det = _calib_tau(scores, 0.35)
    odet, on = O.detect(orc_raw, A, NC, aw, 32, hw, hw, tau_det)
    cap = 64
    m_det = B.Model(det_spec, Bn, params=p_det)
    m_veh = B.Model(veh, cap, params=p_veh)
    m_per = B.Model(per, cap, params=p_per)
    app = B.App([m_det, m_veh, m_per], edges=[(0, 1, B.ROUTE_DET_CROP, 0, crop, crop),
                                               (0, 2, B.ROUTE_DET_CROP, 1, crop, crop)], max_routed_per_dst=cap)
    max_det = Bn * G * G * A
    outs = [B.alloc_outs(m_det, Bn, max_det=max_det, n_out_edges=2, max_routed=cap), B.alloc_outs(m_veh, cap),
            B.alloc_outs(m_per, cap)]
    taus_cls = [0.5]
    app.infer(to_cuda_bf16(xb), [tau_det] + taus_cls + taus_cls, outs)
    torch.cuda.synchronize()
    n_det = int(outs[0]["n_det"].item())
    gdet = outs[0]["det_table"].cpu().numpy()[:n_det]
    # detection set / order bit-exact outside the band
    band = np.abs(scores - tau_det) < BAND

    def key(rows):
        return [tuple(int(v) for v in r[:4]) for r in rows]

    cand_id = lambda r: ((int(r[0]) * G * G + int(r[1])) * A + int(r[2]))
    gk = [k for k, r in zip(key(gdet), gdet) if not band[cand_id(r)]]
    ok = [k for k, r in zip(key(odet), odet) if not band[cand_id(r)]]
    assert gk == ok
    # every candidate detected by one side only is inside the band
    gset, oset = {cand_id(r) for r in gdet}, {cand_id(r) for r in odet}
    assert all(band[c] for c in gset ^ oset)
    assert n_det - on == len(gset - oset) - len(oset - gset)
    # boxes and scores (matched by candidate id)
    omap = {cand_id(r): r for r in odet}
    for r in gdet:
        c = cand_id(r)
        if c in omap and not band[c]:
            o = omap[c]
            # scores and boxes are sigmoid / exp transforms of the head logits: held to the north_star logit
            # tolerance (2e-2 relative; boxes + 0.5 px), reading Q20 as amended in DESIGN.md (the detector's spread
            # logits drift ~6e-3, and the inference-only fused first conv + pool accumulates its 27 taps in fp32)
            assert abs(r[4] - o[4]) <= 2e-2 * o[4], (r[4], o[4])
            size = max(o[7] - o[5], o[8] - o[6], 1.0)
            assert np.all(np.abs(r[5:] - o[5:]) <= 0.5 + 2e-2 * size), (r, o)
    # routing: per class, ascending detection numbers; counts = detections of that class
    n_routed = outs[0]["n_routed"].cpu().numpy()
    ridx = outs[0]["route_idx"].cpu().numpy()
    for e, cls in enumerate((0, 1)):
        want = [i for i in range(n_det) if int(gdet[i][3]) == cls]
        assert n_routed[e] == len(want)
        assert ridx[e][:min(len(want), cap)].tolist() == want[:cap]
    # stage-isolated crops + downstream classifiers: oracle crops from the GPU boxes
    for e, (model_spec, params, mi) in enumerate(((veh, p_veh, 1), (per, p_per, 2))):
        nr = min(int(n_routed[e]), cap)
        if nr == 0:
            continue
        crops = np.stack([O.crop(xf[int(gdet[d][0])], gdet[d][5:9], crop, crop) for d in ridx[e][:nr]])
        # Q20: crops from the GPU's boxes are bit-exact (the routed batch read back through adainf_dbg_app_crops)
        gcrops = synth.bf16_bits_to_f32(app.crops(e, nr).cpu().numpy().view(np.uint16))
        assert np.array_equal(gcrops, crops), np.abs(gcrops - crops).max()
        orc = O.Model(model_spec).forward(params, crops)
        eid, _, _ = O.exit_assign(orc["conf"], taus_cls)
        g_eid = outs[mi]["exit_id"].cpu().numpy()[:nr]
        cband = np.abs(orc["conf"][:, 0] - taus_cls[0]) < BAND
        assert (g_eid[~cband] == eid[~cband]).all()
        lg = outs[mi]["logits"].cpu().numpy()[:nr]
        for r in np.nonzero(~cband)[0]:
            assert rel(lg[r], orc["logits"][r, eid[r]]) <= 2e-2
        cnt = outs[mi]["exit_counts"].cpu().numpy()
        assert cnt.sum() == nr


def test_audio_dag_class_routing():
    """Event classifier -> whole-input routing by predicted class -> keyword / siren classifiers."""
    Bn = 40
    ev, kw, sr = small_cls(2, in_c=1), small_cls(8, in_c=1), small_cls(4, in_c=1)
    pe, pk, ps = synth.init_params(ev, seed=31), synth.init_params(kw, seed=32), synth.init_params(sr, seed=33)
    sb, _ = synth.spectrograms(Bn, num_classes=8, F=32, T=32, seed=3)
    sf = synth.bf16_bits_to_f32(sb)
    orc = O.Model(ev).forward(pe, sf)
    taus = synth.calibrate_thresholds(orc["conf"], [0.5])
    eid, _, _ = O.exit_assign(orc["conf"], taus)
    o_pred = orc["pred"][np.arange(Bn), eid]
    cap = Bn
    me, mk, ms = B.Model(ev, Bn, params=pe), B.Model(kw, cap, params=pk), B.Model(sr, cap, params=ps)
    app = B.App([me, mk, ms], edges=[(0, 1, B.ROUTE_CLASS_WHOLE, 0, 0, 0), (0, 2, B.ROUTE_CLASS_WHOLE, 1, 0, 0)],
                max_routed_per_dst=cap)
    outs = [B.alloc_outs(me, Bn, n_out_edges=2, max_routed=cap), B.alloc_outs(mk, cap), B.alloc_outs(ms, cap)]
    app.infer(to_cuda_bf16(sb), list(taus) + [0.5, 0.5], outs)
    torch.cuda.synchronize()
    g_pred = outs[0]["pred"].cpu().numpy()
    band = np.abs(orc["conf"][:, 0] - taus[0]) < BAND
    srt = np.sort(orc["logits"][np.arange(Bn), eid], axis=1)
    sep = (srt[:, -1] - srt[:, -2]) > 1e-2
    ok = ~band & sep
    assert (g_pred[ok] == o_pred[ok]).all()
    n_routed = outs[0]["n_routed"].cpu().numpy()
    ridx = outs[0]["route_idx"].cpu().numpy()
    for e, (cls, spec, params, mi) in enumerate(((0, kw, pk, 1), (1, sr, ps, 2))):
        want = [i for i in range(Bn) if g_pred[i] == cls]  # routing follows the GPU's own decisions
        assert n_routed[e] == len(want) and ridx[e][:len(want)].tolist() == want
        if not want:
            continue
        o2 = O.Model(spec).forward(params, sf[want])
        e2, _, _ = O.exit_assign(o2["conf"], [0.5])
        b2 = np.abs(o2["conf"][:, 0] - 0.5) < BAND
        g_e2 = outs[mi]["exit_id"].cpu().numpy()[:len(want)]
        assert (g_e2[~b2] == e2[~b2]).all()
        lg = outs[mi]["logits"].cpu().numpy()[:len(want)]
        for r in np.nonzero(~b2)[0]:
            assert rel(lg[r], o2["logits"][r, e2[r]]) <= 2e-2


def test_video_dag_c3_geometry():
    """BASELINE config 3 geometry on a few frames: 416x416 frames, TinyYOLOv3-like detector at G = 13 (stride 32),
    crops resized to 224x224 into two ResNet-18-EE destinations (vehicle 10 classes, person 8 classes), all on
    the device; detections / routing bit-exact outside the tau_det band, crops bit-exact from the GPU's boxes,
    downstream exits and logits against the oracle on those crops."""
    Bn, hw, crop = 3, 416, 224
    det_spec = S.tiny_yolo_det(in_hw=hw)
    A, NC = 3, 2
    p_det = synth.det_head_params(det_spec, synth.init_params(det_spec, seed=51), obj_bias=-1.0)
    veh, per = S.resnet18_ee(10), S.resnet18_ee(8)
    p_veh, p_per = synth.init_params(veh, seed=52), synth.init_params(per, seed=53)
    xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=51)
    xf = synth.bf16_bits_to_f32(xb)
    raw = O.Model(det_spec).forward(p_det, xf, want_det=True)["det"]
    G = raw.shape[1]
    assert G == 13
    sig = lambda v: 1 / (1 + np.exp(-v.astype(np.float64)))
    r5 = raw.reshape(Bn, G, G, A, 5 + NC)
    scores = (sig(r5[..., 4]) * sig(r5[..., 5:].max(-1))).reshape(-1)
    # ~4 detections per frame, threshold in the widest nearby gap
    tau_det = _calib_tau(scores, 4.0 * Bn / scores.size)
    odet, on = O.detect(raw, A, NC, S.YOLO_ANCHORS, 32, hw, hw, tau_det)
    cap = 48
    m_det = B.Model(det_spec, Bn, params=p_det)
    m_veh, m_per = B.Model(veh, cap, params=p_veh), B.Model(per, cap, params=p_per)
    app = B.App([m_det, m_veh, m_per], edges=[(0, 1, B.ROUTE_DET_CROP, 0, crop, crop),
                                               (0, 2, B.ROUTE_DET_CROP, 1, crop, crop)], max_routed_per_dst=cap)
    max_det = Bn * G * G * A
    outs = [B.alloc_outs(m_det, Bn, max_det=max_det, n_out_edges=2, max_routed=cap), B.alloc_outs(m_veh, cap),
            B.alloc_outs(m_per, cap)]
    taus_cls = [0.4, 0.4, 0.4]
    app.infer(to_cuda_bf16(xb), [tau_det] + taus_cls + taus_cls, outs)
    app.poll()
    n_det = int(outs[0]["n_det"].item())
    gdet = outs[0]["det_table"].cpu().numpy()[:n_det]
    band = np.abs(scores - tau_det) < BAND
    cid = lambda r: (int(r[0]) * G * G + int(r[1])) * A + int(r[2])
    assert [tuple(int(v) for v in r[:4]) for r in gdet if not band[cid(r)]] == \
        [tuple(int(v) for v in r[:4]) for r in odet if not band[cid(r)]]
    assert 1 <= n_det <= cap
    n_routed = outs[0]["n_routed"].cpu().numpy()
    ridx = outs[0]["route_idx"].cpu().numpy()
    assert int(n_routed.sum()) == n_det
    for e, (model_spec, params, mi, taus) in enumerate(((veh, p_veh, 1, taus_cls), (per, p_per, 2, taus_cls))):
        want = [i for i in range(n_det) if int(gdet[i][3]) == e]
        assert n_routed[e] == len(want) and ridx[e][:len(want)].tolist() == want
        nr = len(want)
        if nr == 0:
            continue
        crops = np.stack([O.crop(xf[int(gdet[d][0])], gdet[d][5:9], crop, crop) for d in want])
        gcrops = synth.bf16_bits_to_f32(app.crops(e, nr).cpu().numpy().view(np.uint16))
        assert np.array_equal(gcrops, crops)
        orc = O.Model(model_spec).forward(params, crops)
        eid, _, counts = O.exit_assign(orc["conf"], taus)
        from parity import banded_rows
        cb = banded_rows(orc["conf"], taus, eid)
        g_eid = outs[mi]["exit_id"].cpu().numpy()[:nr]
        assert (g_eid[~cb] == eid[~cb]).all()
        assert outs[mi]["exit_counts"].cpu().numpy().sum() == nr
        lg = outs[mi]["logits"].cpu().numpy()[:nr]
        for r in np.nonzero(~cb)[0]:
            assert rel(lg[r], orc["logits"][r, eid[r]]) <= 2e-2
    app.close()
    for m in (m_det, m_veh, m_per):
        m.close()


def test_detector_nms_stage_isolated():
    """NEXT-3 (reading Q18b): greedy per-(frame, class) NMS on the device between decode and routing.  Stage
    isolation as for the crops (Q20): the same detector without NMS yields the GPU's pre-NMS detections; the oracle's
    NMS on exactly those rows must select exactly the rows the NMS-enabled detector keeps (bit-exact, in order), and
    routing must list the kept rows by class."""
    Bn, hw = 3, 416
    base = S.tiny_yolo_det(in_hw=hw)
    nmsd = S.tiny_yolo_det(in_hw=hw, nms_iou=0.45)
    A, NC = 3, 2
    p = synth.det_head_params(base, synth.init_params(base, seed=61), obj_bias=-1.0)
    xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=61)
    x = to_cuda_bf16(xb)
    G = hw // 32
    max_det = Bn * G * G * A
    res = {}
    for name, spec in (("pre", base), ("nms", nmsd)):
        m = B.Model(spec, Bn, params=p)
        veh, per = small_cls(10, hw=32), small_cls(8, hw=32)
        mv, mp = B.Model(veh, max_det, params=synth.init_params(veh, seed=62)), B.Model(per, max_det,
                                                                                    params=synth.init_params(per, seed=63))
        app = B.App([m, mv, mp], edges=[(0, 1, B.ROUTE_DET_CROP, 0, 32, 32), (0, 2, B.ROUTE_DET_CROP, 1, 32, 32)],
                    max_routed_per_dst=max_det)
        outs = [B.alloc_outs(m, Bn, max_det=max_det, n_out_edges=2, max_routed=max_det), B.alloc_outs(mv, max_det),
                B.alloc_outs(mp, max_det)]
        app.infer(x, [0.12] + [0.5] + [0.5], outs)
        app.poll()
        n = int(outs[0]["n_det"].item())
        res[name] = (outs[0]["det_table"].cpu().numpy()[:n].copy(), outs[0]["n_routed"].cpu().numpy().copy(),
                     outs[0]["route_idx"].cpu().numpy().copy())
        app.close()
        for mm in (m, mv, mp):
            mm.close()
    pre, _, _ = res["pre"]
    got, n_routed, ridx = res["nms"]
    assert pre.shape[0] > 50  # plenty of overlapping candidates per frame
    keep, nk = O.nms(pre, 0.45)
    assert 0 < nk < pre.shape[0]
    np.testing.assert_array_equal(got, pre[keep.astype(bool)])
    for e in range(2):
        want = [i for i in range(got.shape[0]) if int(got[i][3]) == e]
        assert n_routed[e] == len(want) and ridx[e][:len(want)].tolist() == want
