"""The bench replays one captured CUDA graph of the whole hot-path step (early-exit inference, retraining
step).  The graph must be a faithful recording of the eagerly launched C-ABI calls: replaying it from the same
model state (after one identical eager warm-up step) gives bit-identical exit decisions, predictions, losses and updated weights, and replaying it
again continues from the updated state exactly like a second eager step."""
import numpy as np
import pytest
import torch

from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

pytestmark = pytest.mark.gpu


def _setup(spec, p, nb, nk):
    m = B.Model(spec, max(nb, nk), params=p)
    app = B.App([m])
    outs = B.alloc_outs(m, nb)
    stats = torch.zeros(2, dtype=torch.float32, device="cuda")
    return m, app, outs, stats


@pytest.mark.parametrize("spec_name,hw", [("resnet18_ee", 224), ("tiny_cnn_ee", 32)])
def test_graph_replay_matches_eager(spec_name, hw):
    spec = getattr(S, spec_name)()
    nb, nk = 48, 64
    p = synth.init_params(spec, seed=7)
    xb, y = synth.drifted_images(nk, hw, hw, 3, seed=7)
    x = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    lab = torch.from_numpy(y).cuda()
    n_exits = sum(op["kind"] == "exit" for op in spec["ops"])
    taus = [0.4] * (n_exits - 1)

    def step(app, m, outs, stats):
        app.infer(x[:nb], taus, [outs])
        m.retrain_step(x[:nk], lab[:nk], lr=0.05, stats=stats)

    # both models take one identical eager step first (first calls allocate workspaces, which a capture
    # must not do), then the eager model takes two more steps and the other replays the captured step twice
    m1, app1, outs1, st1 = _setup(spec, p, nb, nk)
    step(app1, m1, outs1, st1)
    eager = []
    for _ in range(2):
        step(app1, m1, outs1, st1)
        torch.cuda.synchronize()
        eager.append((outs1["exit_id"].clone(), outs1["pred"].clone(), st1.clone(), m1.get_params().copy()))
    # graph: capture (does not execute), replay twice from the same initial state
    m2, app2, outs2, st2 = _setup(spec, p, nb, nk)
    step(app2, m2, outs2, st2)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step(app2, m2, outs2, st2)
    torch.cuda.synchronize()
    for k in range(2):
        g.replay()
        torch.cuda.synchronize()
        e_id, e_pred, e_st, e_par = eager[k]
        assert torch.equal(outs2["exit_id"], e_id)
        assert torch.equal(outs2["pred"], e_pred)
        assert torch.equal(st2, e_st)
        assert np.array_equal(m2.get_params(), e_par)
