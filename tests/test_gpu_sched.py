"""Incremental-retraining support on the GPU (include/adainf_sched.h, driver.py):
version averaging, disjoint-sample marking, prediction counts, and one job of the
retraining -> inference DAG whose selections match the oracle and never overlap between jobs."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import driver as D
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import to_cuda_bf16

pytestmark = pytest.mark.gpu


def test_model_average_is_ordered_fp32_mean_and_resets_momentum():
    spec = S.tiny_cnn_ee()
    ps = [synth.init_params(spec, seed=s) for s in (1, 2, 3)]
    ms = [B.Model(spec, 64, params=p) for p in ps]
    xb, y = synth.drifted_images(64, 32, 32, 3, seed=9)
    x, yt = to_cuda_bf16(xb), torch.from_numpy(y).cuda()
    ms[0].retrain_step(x, yt, lr=0.05)  # gives model 0 a nonzero momentum
    p0 = ms[0].get_params()
    B.model_average(ms[0], ms)
    torch.cuda.synchronize()
    acc = p0.copy()
    acc += ps[1]
    acc += ps[2]
    expect = acc / np.float32(3)
    got = ms[0].get_params()
    assert np.array_equal(got, expect)
    # momentum reset: one step from the average equals one step of a fresh model holding the average
    ref = B.Model(spec, 64, params=expect)
    ms[0].retrain_step(x, yt, lr=0.05)
    ref.retrain_step(x, yt, lr=0.05)
    assert np.array_equal(ms[0].get_params(), ref.get_params())
    for m in ms + [ref]:
        m.close()


def test_mark_used_and_count_correct():
    ex = torch.zeros(1000, dtype=torch.uint8, device="cuda")
    idx = torch.tensor([3, 999, 10, 500], dtype=torch.int32, device="cuda")
    cnt = torch.tensor([3], dtype=torch.int32, device="cuda")
    B.mark_used(ex, idx, cnt)
    e = ex.cpu().numpy()
    assert e.sum() == 3 and e[3] == e[999] == e[10] == 1 and e[500] == 0
    pred = torch.tensor([1, 2, 3, 4, 5], dtype=torch.int32, device="cuda")
    lab = torch.tensor([1, 0, 3, 4, 0], dtype=torch.int32, device="cuda")
    assert int(B.count_correct(pred, lab).item()) == 3


def test_run_job_retrain_then_infer_disjoint_selections():
    spec = S.tiny_cnn_ee()
    p = synth.init_params(spec, seed=5)
    N, Dm, P = 2048, 64, 16
    xb, y = synth.drifted_images(N, 32, 32, 3, seed=11)
    Xb, Wb, ref = synth.embeddings(N, Dm, P, seed=11)
    pool_x, pool_y = to_cuda_bf16(xb), torch.from_numpy(y).cuda()
    emb = torch.from_numpy(Xb.view(np.int16)).cuda().view(torch.bfloat16).reshape(N, Dm)
    W = torch.from_numpy(Wb.view(np.int16)).cuda().view(torch.bfloat16).reshape(Dm, P)
    R = torch.from_numpy(ref).cuda()
    exclude = torch.zeros(N, dtype=torch.uint8, device="cuda")
    m = B.Model(spec, 256, params=p)
    app = B.App([m])
    req, _ = synth.drifted_images(64, 32, 32, 3, seed=12)
    req = to_cuda_bf16(req)
    outs = B.alloc_outs(m, 64)
    batches = [64, 128, 256]
    step_ms = D.profile_retrain(m, pool_x, pool_y, batches)
    inf_ms = D.profile_infer(app, req, [0.5], outs)
    assert all(t > 0 for t in step_ms) and inf_ms > 0
    sel_idx = torch.empty(N, dtype=torch.int32, device="cuda")
    sel_cnt = torch.empty(1, dtype=torch.int32, device="cuda")
    rt_x = torch.empty((256, 32, 32, 3), dtype=torch.bfloat16, device="cuda")
    rt_y = torch.empty(256, dtype=torch.int32, device="cuda")
    task = D.RetrainTask(model=m, impact=0.1, pool_x=pool_x, pool_y=pool_y, emb=emb, pca=W, ref=R,
                         exclude=exclude, eligible=N, lr=0.02, profile_batches=batches, profile_ms=step_ms)
    # an SLO leaving room for a few steps of the largest batch
    slo = inf_ms + 3.5 * step_ms[-1]
    rep = D.run_job(app, req, [0.5], outs, slo, [inf_ms], [task], sel_idx, sel_cnt, rt_x, rt_y)
    plan = rep["plans"][0]
    assert rep["spare_ms"] == pytest.approx(slo - inf_ms)
    assert plan["steps"] >= 1 and plan["samples"] >= 64
    Rn = plan["samples"]
    first = sel_idx[:Rn].cpu().numpy().copy()
    assert int(exclude.sum().item()) == Rn
    # the selection is the oracle's top-R by cosine distance outside the decision band
    oi, _, oc, odist = O.select(synth.bf16_bits_to_f32(Xb).reshape(N, Dm), synth.bf16_bits_to_f32(Wb).reshape(Dm, P),
                                ref, Rn)
    dk = np.sort(odist)[::-1][Rn - 1]
    band = np.abs(odist - dk) < 1e-3
    assert set(i for i in first.tolist() if not band[i]) == set(i for i in oi.tolist() if not band[i])
    assert not np.array_equal(m.get_params(), p)  # the model was retrained before inference
    assert int(outs["exit_counts"].sum().item()) == 64
    # the next job of the application: disjoint samples
    rep2 = D.run_job(app, req, [0.5], outs, slo, [inf_ms], [task], sel_idx, sel_cnt, rt_x, rt_y)
    R2 = rep2["plans"][0]["samples"]
    second = sel_idx[:R2].cpu().numpy()
    assert not set(first.tolist()) & set(second.tolist())
    assert int(exclude.sum().item()) == Rn + R2
    app.close()
    m.close()


def test_detect_drift_full_structure_accuracy_and_stop_rule():
    """NEXT-2: two models of an application; I'_m on the S most divergent samples with the full
    structure matches the oracle's prediction count on the same samples; a model whose initial accuracy is
    above I'_m is impacted, one with I_m = 0 never is; the impacted set is constant, so the process stops after
    4 values of S (3%..12%)."""
    spec = S.tiny_cnn_ee()
    N, Dm, P = 1024, 64, 16
    xb, y = synth.drifted_images(N, 32, 32, 3, seed=21)
    Xb, Wb, ref = synth.embeddings(N, Dm, P, seed=21)
    pool_x, pool_y = to_cuda_bf16(xb), torch.from_numpy(y).cuda()
    emb = torch.from_numpy(Xb.view(np.int16)).cuda().view(torch.bfloat16).reshape(N, Dm)
    W = torch.from_numpy(Wb.view(np.int16)).cuda().view(torch.bfloat16).reshape(Dm, P)
    R = torch.from_numpy(ref).cuda()
    dms, params = [], []
    for seed, i_m in ((31, 0.95), (32, 0.0)):
        p = synth.init_params(spec, seed=seed)
        params.append(p)
        m = B.Model(spec, 256, params=p)
        dms.append(D.DriftModel(app=B.App([m]), model=m, initial_acc=i_m, emb=emb, pca=W, ref=R, pool_x=pool_x,
                                pool_y=pool_y))
    mask, degrees, trace = D.detect_drift(dms)
    assert mask == 0b01
    assert [t["fraction"] for t in trace] == [0.03, 0.06, 0.09, 0.12]
    # I'_m at the last S against the oracle on the oracle's own selection of the same S samples
    Sn = int(round(0.12 * N))
    oi, _, _, _ = O.select(synth.bf16_bits_to_f32(Xb).reshape(N, Dm), synth.bf16_bits_to_f32(Wb).reshape(Dm, P), ref, Sn)
    for j, p in enumerate(params):
        orc = O.Model(spec).forward(p, synth.bf16_bits_to_f32(xb[oi]))
        o_acc = float((orc["pred"][:, -1] == y[oi]).mean())
        assert abs(trace[-1]["acc"][j] - o_acc) <= 2.0 / Sn, (j, trace[-1]["acc"][j], o_acc)
        assert degrees[j] == pytest.approx(dms[j].initial_acc - trace[-1]["acc"][j])
    for dm in dms:
        dm.app.close()
        dm.model.close()


def test_next4_structure_profiles_and_choice():
    """NEXT-4 on the B200: per-(structure, batch) latency table of ResNet-18-EE measured with CUDA events, the
    structures' accuracies counted on the device, and the structure / batch choice equal to brute
    force over the same measured tables."""
    from paper_conf_sigcomm_shubhas23_b200 import driver as D
    spec = S.resnet18_ee(in_hw=64)
    p = synth.init_params(spec, seed=3)
    xb, y = synth.drifted_images(64, 64, 64, 3, seed=3)
    x = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    yt = torch.from_numpy(y).cuda()
    m = B.Model(spec, 64, params=p)
    app = B.App([m])
    outs = B.alloc_outs(m, 64)
    structs = D.early_exit_structures(4)
    batches = [8, 16, 32, 64]
    tables = D.profile_structures(app, x, structs, batches, outs, reps=3)
    assert all(t > 0 for row in tables for t in row)
    # truncating at exit 0 runs the stem + layer 1 only: faster than the full structure at every batch
    assert all(a < f for a, f in zip(tables[0], tables[-1]))
    acc = D.structure_accuracy(app, x, yt, structs, outs)
    assert all(0.0 <= a <= 1.0 for a in acc)
    for a_min in (0.0, sorted(acc)[1], 2.0):
        s, b, w = D.plan_inference(batches, tables, acc, a_min, True, 100)
        b0 = min(batches, key=lambda bb: (tables[-1][batches.index(bb)] * -(-100 // bb), bb))
        ok = [i for i in range(4) if acc[i] >= a_min]
        want = min(ok, key=lambda i: (tables[i][batches.index(b0)], i)) if ok else 3
        assert s == want
        ws = [tables[s][i] * -(-100 // bb) for i, bb in enumerate(batches)]
        assert w == min(ws) and b == batches[ws.index(min(ws))]
    app.close()
    m.close()
