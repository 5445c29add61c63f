"""Edge cases of this round's paths (empty, single-row and ragged batches): a detector DAG routing NOTHING to
MobileNetV2 / ShuffleNet / conv+pool destinations (every device count 0, nothing written, no fault), the same DAG
routing EVERY candidate (capacity clamp in candidate order, the overflow reported by poll), and single-row / ragged
(129 = 128 + 1 rows) batches of the new model families against the oracle."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import bn_folded_params, check_infer_parity, gpu_infer_single, images, rel, to_cuda_bf16
from test_gpu_dag import small_cls
from test_gpu_mnv2 import mnv2_blocks_spec
from test_gpu_shufflenet import shuffle_units_spec

pytestmark = pytest.mark.gpu


def _dsts(which, crop):
    sh = dict(shuffle_units_spec(hw=crop), in_w=crop)  # square input: crops are crop x crop
    return {"mnv2_shuffle": [mnv2_blocks_spec(hw=crop), sh],
            "cnn_mnv2": [small_cls(5, hw=crop), mnv2_blocks_spec(hw=crop)]}[which]


def _dag(tau_det, cap, which):
    Bn, hw, crop = 3, 96, 32
    det = S.tiny_yolo_det(in_hw=hw, nms_iou=0.45)
    p_det = synth.det_head_params(det, synth.init_params(det, seed=41), obj_bias=0.0)
    dsts = _dsts(which, crop)
    ms = [B.Model(det, Bn, params=p_det)] + [B.Model(s, cap, params=synth.init_params(s, seed=42 + i))
                                              for i, s in enumerate(dsts)]
    # detector class 0 / 1 -> destination 1 / 2 (one destination per class)
    edges = [(0, 1, B.ROUTE_DET_CROP, 0, crop, crop), (0, 2, B.ROUTE_DET_CROP, 1, crop, crop)]
    app = B.App(ms, edges=edges, max_routed_per_dst=cap)
    G = hw // 32
    max_det = Bn * G * G * 3
    outs = [B.alloc_outs(ms[0], Bn, max_det=max_det, n_out_edges=2, max_routed=cap)] + \
           [B.alloc_outs(m, cap) for m in ms[1:]]
    xb, _ = synth.drifted_images(Bn, hw, hw, 3, seed=41)
    taus = [tau_det] + [0.5] + [0.5]
    return app, ms, outs, xb, taus


def _close(app, ms):
    app.close()
    for m in ms:
        m.close()


@pytest.mark.parametrize("which", ["mnv2_shuffle", "cnn_mnv2"])
def test_dag_routes_nothing(which):
    app, ms, outs, xb, taus = _dag(2.0, 16, which)
    app.infer(to_cuda_bf16(xb), taus, outs)
    app.poll()
    torch.cuda.synchronize()
    assert int(outs[0]["n_det"].item()) == 0
    assert outs[0]["n_routed"].cpu().numpy().tolist() == [0, 0]
    for o in outs[1:]:
        assert int(o["exit_counts"].sum().item()) == 0
        assert (o["exit_id"].cpu().numpy() == -1).all()  # nothing written
    _close(app, ms)


@pytest.mark.parametrize("which", ["mnv2_shuffle", "cnn_mnv2"])
def test_dag_routes_everything_with_capacity_clamp(which):
    cap = 4
    app, ms, outs, xb, taus = _dag(0.0, cap, which)  # tau_det = 0: every candidate is a detection (then NMS)
    app.infer(to_cuda_bf16(xb), taus, outs)
    with pytest.raises(B.AdaInfError) as ei:
        app.poll()
    assert ei.value.code == B.ERR_CAPACITY
    torch.cuda.synchronize()
    n_det = int(outs[0]["n_det"].item())
    det = outs[0]["det_table"].cpu().numpy()[:n_det]
    n_routed = outs[0]["n_routed"].cpu().numpy()
    ridx = outs[0]["route_idx"].cpu().numpy()
    for e in range(2):
        want = [i for i in range(n_det) if int(det[i][3]) == e]
        assert n_routed[e] == len(want) > cap  # the required count is reported
        assert ridx[e][:cap].tolist() == want[:cap]  # clamped in candidate order
        assert int(outs[1 + e]["exit_counts"].sum().item()) == cap
    _close(app, ms)


def test_two_edges_for_one_class_are_rejected():
    det = S.tiny_yolo_det(in_hw=64)
    ms = [B.Model(det, 2), B.Model(small_cls(5), 4), B.Model(small_cls(3), 4)]
    with pytest.raises(B.AdaInfError) as ei:
        B.App(ms, edges=[(0, 1, B.ROUTE_DET_CROP, 0, 32, 32), (0, 2, B.ROUTE_DET_CROP, 0, 32, 32)],
              max_routed_per_dst=4)
    assert ei.value.code == B.ERR_INVALID
    for m in ms:
        m.close()


@pytest.mark.parametrize("which,Bn", [("shuffle", 1), ("shuffle", 129), ("mnv2", 1), ("mnv2", 129)])
def test_single_and_ragged_batches(which, Bn):
    spec = shuffle_units_spec() if which == "shuffle" else mnv2_blocks_spec()
    xb, _, xf = images(spec, Bn, 43)
    p = synth.init_params(spec, seed=43)
    calib = images(spec, 48, 44)[2]  # the input recipe's statistics from a separate batch
    p = bn_folded_params(spec, p, calib)
    p = synth.spread_exit_heads(spec, p, O.Model(spec).forward(p, calib)["logits"])
    orc = O.Model(spec).forward(p, xf)
    taus = [0.5]
    gpu = gpu_infer_single(spec, p, xb, taus)
    check_infer_parity(orc, gpu, taus)
    g_full = gpu_infer_single(spec, p, xb, [2.0])
    for r in range(Bn):
        assert rel(g_full["logits"][r], orc["logits"][r, 1]) <= 2e-2
