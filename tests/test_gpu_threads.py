"""C-ABI thread-safety contract (include/adainf.h): distinct model handles are independent, so two host
threads driving two models on two streams at once must produce exactly what the same calls produce one after
the other (the library's host-side kernel-parameter staging is per thread)."""
import threading

import numpy as np
import pytest
import torch

from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

pytestmark = pytest.mark.gpu


def _job(seed, n=32, steps=2):
    spec = S.resnet18_ee()
    p = synth.init_params(spec, seed=seed)
    xb, y = synth.drifted_images(n, 224, 224, 3, seed=seed)
    x = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.bfloat16)
    lab = torch.from_numpy(y).cuda()
    m = B.Model(spec, n, params=p)
    app = B.App([m])
    outs = B.alloc_outs(m, n)
    return m, app, outs, x, lab, steps


def _run(job, stream):
    m, app, outs, x, lab, steps = job
    with torch.cuda.stream(stream):
        for _ in range(steps):
            app.infer(x, [0.4, 0.3, 0.3], [outs])
            m.retrain_step(x, lab, lr=0.05)
    stream.synchronize()
    return outs["exit_id"].cpu().clone(), outs["pred"].cpu().clone(), m.get_params().copy()


def test_two_models_two_threads_match_sequential():
    seq = [_run(_job(s), torch.cuda.Stream()) for s in (11, 12)]
    jobs = [_job(s) for s in (11, 12)]
    res = [None, None]

    def worker(i):
        res[i] = _run(jobs[i], torch.cuda.Stream())

    th = [threading.Thread(target=worker, args=(i,)) for i in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for i in range(2):
        assert torch.equal(res[i][0], seq[i][0])
        assert torch.equal(res[i][1], seq[i][1])
        assert np.array_equal(res[i][2], seq[i][2])
