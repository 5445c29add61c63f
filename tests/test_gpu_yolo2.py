"""NEXT-3 on the GPU: the two-scale TinyYOLOv3-like detector (reading Q18c) — ROUTE back to the 13x13 1x1 conv,
1x1 conv, x2 nearest upsample read through the concat with the 26x26 feature map, the second (stride-16) head, both
scales decoded into one candidate order (the second head's cells after the first's in each frame) and NMS'd together
— against the oracle: the detection set / order bit-exact outside the tau_det band, scores and boxes within the
north_star logit tolerance, and the NMS stage-isolated (the oracle's NMS on the GPU's own pre-NMS rows selects
exactly the rows the NMS-enabled detector keeps)."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import BAND, to_cuda_bf16
from test_gpu_dag import _calib_tau, small_cls

pytestmark = pytest.mark.gpu
A, NC = 3, 2


def _run(spec, p, xb, tau_det, max_det):
    Bn, hw = xb.shape[0], spec["in_h"]
    m = B.Model(spec, Bn, params=p)
    veh, per = small_cls(10, hw=32), small_cls(8, hw=32)
    mv = B.Model(veh, max_det, params=synth.init_params(veh, seed=92))
    mp = B.Model(per, max_det, params=synth.init_params(per, seed=93))
    app = B.App([m, mv, mp], edges=[(0, 1, B.ROUTE_DET_CROP, 0, 32, 32), (0, 2, B.ROUTE_DET_CROP, 1, 32, 32)],
                max_routed_per_dst=max_det)
    outs = [B.alloc_outs(m, Bn, max_det=max_det, n_out_edges=2, max_routed=max_det), B.alloc_outs(mv, max_det),
            B.alloc_outs(mp, max_det)]
    app.infer(to_cuda_bf16(xb), [tau_det, 0.5, 0.5], outs)
    app.poll()
    n = int(outs[0]["n_det"].item())
    r = (outs[0]["det_table"].cpu().numpy()[:n].copy(), outs[0]["n_routed"].cpu().numpy().copy(),
         outs[0]["route_idx"].cpu().numpy().copy())
    app.close()
    for mm in (m, mv, mp):
        mm.close()
    return r


def test_two_scale_decode_vs_oracle():
    Bn, hw = 6, 96
    spec = S.tiny_yolo_det2(in_hw=hw, nms_iou=0.0)
    p = synth.det_head_params(spec, synth.init_params(spec, seed=91), obj_bias=0.0)
    xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=91)
    xf = synth.bf16_bits_to_f32(xb)
    raws = O.Model(spec).forward(p, xf, want_det=True)["det"]
    assert len(raws) == 2 and raws[0].shape[1] == hw // 32 and raws[1].shape[1] == hw // 16
    G0, G1 = raws[0].shape[1], raws[1].shape[1]
    cpf = G0 * G0 + G1 * G1
    sig = lambda v: 1 / (1 + np.exp(-v.astype(np.float64)))
    # scores in candidate order (frame, head-0 cells, head-1 cells, anchor)
    sc = [(sig(r.reshape(Bn, -1, A, 5 + NC)[..., 4]) * sig(r.reshape(Bn, -1, A, 5 + NC)[..., 5:].max(-1)))
          for r in raws]
    scores = np.concatenate(sc, axis=1).reshape(-1)
    tau = _calib_tau(scores, 0.35)
    odet, on = O.detect_multi(raws, A, NC, [S.YOLO_ANCHORS, S.YOLO_ANCHORS_26], [32, 16], hw, hw, tau)
    max_det = Bn * cpf * A
    gdet, n_routed, ridx = _run(spec, p, xb, tau, max_det)
    band = np.abs(scores - tau) < BAND
    cand = lambda r: (int(r[0]) * cpf + int(r[1])) * A + int(r[2])
    gk = [tuple(int(v) for v in r[:4]) for r in gdet if not band[cand(r)]]
    ok = [tuple(int(v) for v in r[:4]) for r in odet if not band[cand(r)]]
    assert gk == ok and len(gk) > 10
    assert any(int(r[1]) >= G0 * G0 for r in gdet) and any(int(r[1]) < G0 * G0 for r in gdet)  # both scales fire
    gset, oset = {cand(r) for r in gdet}, {cand(r) for r in odet}
    assert all(band[c] for c in gset ^ oset)
    omap = {cand(r): r for r in odet}
    for r in gdet:
        c = cand(r)
        if c in omap and not band[c]:
            o = omap[c]
            assert abs(r[4] - o[4]) <= 2e-2 * o[4], (r[4], o[4])
            size = max(o[7] - o[5], o[8] - o[6], 1.0)
            assert np.all(np.abs(r[5:] - o[5:]) <= 0.5 + 2e-2 * size), (r, o)
    for e in range(2):
        want = [i for i in range(gdet.shape[0]) if int(gdet[i][3]) == e]
        assert n_routed[e] == len(want) and ridx[e][:len(want)].tolist() == want


def test_two_scale_nms_stage_isolated():
    Bn, hw = 2, 416
    base = S.tiny_yolo_det2(in_hw=hw, nms_iou=0.0)
    nmsd = S.tiny_yolo_det2(in_hw=hw, nms_iou=0.45)
    p = synth.det_head_params(base, synth.init_params(base, seed=94), obj_bias=-1.0)
    xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=94)
    max_det = Bn * (13 * 13 + 26 * 26) * A
    pre, _, _ = _run(base, p, xb, 0.12, max_det)
    got, n_routed, ridx = _run(nmsd, p, xb, 0.12, max_det)
    assert pre.shape[0] > 100 and (pre[:, 1] >= 169).any()
    keep, nk = O.nms(pre, 0.45)
    assert 0 < nk < pre.shape[0]
    np.testing.assert_array_equal(got, pre[keep.astype(bool)])
    for e in range(2):
        want = [i for i in range(got.shape[0]) if int(got[i][3]) == e]
        assert n_routed[e] == len(want) and ridx[e][:len(want)].tolist() == want


def test_two_scale_detector_is_inference_only():
    spec = S.tiny_yolo_det2(in_hw=64)
    m = B.Model(spec, 2)
    x = torch.zeros(2, 64, 64, 3, dtype=torch.bfloat16, device="cuda")
    with pytest.raises(B.AdaInfError) as ei:
        m.retrain_step(x, torch.zeros(2, dtype=torch.int32, device="cuda"), lr=0.0)
    assert ei.value.code == B.ERR_UNSUPPORTED
    m.close()
