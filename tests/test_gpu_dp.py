"""libadainf's data-parallel retraining path on the one GPU of the
box: world-2 process groups over gloo, each rank a separate process with its own adainf model on cuda:0.

Each rank computes its disjoint shard's gradient (index mod G, scaled by 1/N_global) with adainf_retrain_grad,
the ranks sum the device gradient buffers (adainf_model_grad_ptr) with a gloo all-reduce, and each applies
adainf_model_update.  Checked: replicas bit-identical after two steps, equal to the single-process full-batch
step (weights within 1e-3 rel, SGD update within 2e-2), adainf_retrain_step == retrain_grad + update bit for
bit, and the same through adainf_retrain_grad_rows with a device count (NCCL itself needs one GPU per rank,
so the NCCL communicator is exercised by bench.py --gpus N on multi-GPU boxes only)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sigcomm_shubhas23_b200 import binding as B
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth

from parity import rel, to_cuda_bf16

pytestmark = pytest.mark.gpu

N, LR = 24, 0.05


def _spec():
    return S.resnet18_ee(in_hw=64)


def _data():
    spec = _spec()
    p = synth.init_params(spec, seed=12)
    xb, y = synth.drifted_images(N, 64, 64, 3, seed=12)
    return spec, p, xb, y


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        spec, p, xb, y = _data()
        idx = np.arange(N)[np.arange(N) % world == rank]
        m = B.Model(spec, len(idx), params=p, momentum=0.9)
        pool = to_cuda_bf16(xb)
        labels = torch.from_numpy(y).cuda()
        for step in range(2):
            if step == 0:
                m.retrain_grad(pool[torch.from_numpy(idx).cuda()].contiguous(),
                               labels[torch.from_numpy(idx).cuda()].contiguous(), n_global=N)
            else:  # the row-mapped variant with a device count
                ridx = torch.from_numpy(idx.astype(np.int32)).cuda()
                cnt = torch.tensor([len(idx)], dtype=torch.int32, device="cuda")
                m.retrain_grad_rows(pool, labels, ridx, n_global=N, count=cnt)
            torch.cuda.synchronize()
            g = m.grad_tensor()
            h = g.cpu()
            dist.all_reduce(h)  # gloo sum of the 1/N-scaled shard gradients
            g.copy_(h.cuda())
            m.update(lr=LR)
            torch.cuda.synchronize()
        q.put((rank, m.get_params()))
        m.close()
        dist.destroy_process_group()
    except Exception as ex:  # pragma: no cover
        q.put((rank, repr(ex)))


def test_dp_world2_gloo_over_libadainf():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=600) for _ in range(2))
    for pr in procs:
        pr.join(timeout=60)
    assert all(isinstance(v, np.ndarray) for v in res.values()), res
    assert np.array_equal(res[0], res[1]), "replicas diverged"
    # single-process full batch, two steps
    spec, p, xb, y = _data()
    m = B.Model(spec, N, params=p, momentum=0.9)
    for _ in range(2):
        m.retrain_step(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), n_global=N, lr=LR)
    full = m.get_params()
    m.close()
    assert rel(res[0], full) <= 1e-3
    assert rel(res[0] - p, full - p) <= 2e-2


def test_retrain_step_equals_grad_plus_update():
    spec, p, xb, y = _data()
    outs = []
    for split in (False, True):
        m = B.Model(spec, N, params=p, momentum=0.9)
        st = torch.zeros(2, dtype=torch.float32, device="cuda")
        for _ in range(2):
            if split:
                m.retrain_grad(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), stats=st)
                m.update(lr=LR, stats=st)
            else:
                m.retrain_step(to_cuda_bf16(xb), torch.from_numpy(y).cuda(), lr=LR, stats=st)
        torch.cuda.synchronize()
        outs.append((m.get_params(), st.cpu().numpy()))
        m.close()
    assert np.array_equal(outs[0][0], outs[1][0])
    assert np.array_equal(outs[0][1], outs[1][1])


def test_update_without_gradient_is_an_error():
    spec, p, _, _ = _data()
    m = B.Model(spec, 4, params=p)
    with pytest.raises(B.AdaInfError) as ei:
        m.update(lr=0.1)
    assert ei.value.code == B.ERR_INVALID
    m.close()


def test_retrain_rows_count_and_out_of_range_rows_contribute_nothing():
    """rows at or past the device count, pool indices outside [0, pool_rows) and labels outside
    [0, num_classes) contribute zero loss and gradient (select_retrain's out_idx tail is never read as a row)."""
    spec, p, xb, y = _data()
    pool = to_cuda_bf16(xb)
    labels = torch.from_numpy(y).cuda()
    valid = [3, 17, 0, 22, 8, 11]
    idx = torch.tensor(valid + [5, -7, 10 ** 6, 9], dtype=torch.int32, device="cuda")  # tail past the count
    cnt = torch.tensor([len(valid)], dtype=torch.int32, device="cuda")
    m = B.Model(spec, idx.numel(), params=p)
    m.retrain_grad_rows(pool, labels, idx, n_global=20, count=cnt)
    g_rows = m.get_grads()
    m.close()
    m = B.Model(spec, len(valid), params=p)
    vi = torch.tensor(valid, device="cuda").long()
    m.retrain_grad(pool[vi].contiguous(), labels[vi].contiguous(), n_global=20)
    g_ref = m.get_grads()
    m.close()
    assert rel(g_rows, g_ref) <= 1e-5
    # out-of-range indices inside the count and ignored labels: same gradient as the valid rows alone
    idx2 = torch.tensor(valid + [-1, 10 ** 6], dtype=torch.int32, device="cuda")
    lab2 = labels.clone()
    lab2[5] = 99  # row 5 gets an out-of-range label
    m = B.Model(spec, idx2.numel() + 1, params=p)
    m.retrain_grad_rows(pool, lab2, torch.cat([idx2, torch.tensor([5], dtype=torch.int32, device="cuda")]),
                        n_global=20)
    g2 = m.get_grads()
    m.close()
    assert rel(g2, g_ref) <= 1e-5


def _sel_worker(rank, world, port, mode, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        N, D, P, k = 8192, 64, 16, 700
        Xb, Wb, ref = synth.embeddings(N, D, P, seed=17)
        ex = (np.random.default_rng(17).random(N) < 0.1).astype(np.uint8)
        rows = np.arange(N)[rank::world] if mode == "mod" else np.arange(N).reshape(world, -1)[rank]
        X = torch.from_numpy(Xb.reshape(N, D)[rows].view(np.int16)).cuda().view(torch.bfloat16)
        W = torch.from_numpy(Wb.view(np.int16)).cuda().view(torch.bfloat16).reshape(D, P)
        e = torch.from_numpy(ex[rows]).cuda()
        idx, dd, cnt = B.select_retrain_sharded(X, W, torch.from_numpy(ref).cuda(), k, dist.group.WORLD, exclude=e,
                                                mode=mode, n_total=N)
        torch.cuda.synchronize()
        c = int(cnt.item())
        q.put((rank, (idx.cpu().numpy()[:c].copy(), dd.cpu().numpy()[:c].copy())))
        dist.destroy_process_group()
    except Exception as ex_:  # pragma: no cover
        q.put((rank, repr(ex_)))


@pytest.mark.parametrize("mode", ["contiguous", "mod"])
def test_sharded_selection_k12_equals_single_gpu(mode):
    """K12: per-shard exact top-k + all-gather + adainf_select_merge == adainf_select_retrain on the
    whole pool, bit for bit (index set, order, distances), for contiguous and index-mod-G shards."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sel_worker, args=(r, 2, port, mode, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=600) for _ in range(2))
    for pr in procs:
        pr.join(timeout=60)
    assert all(isinstance(v, tuple) for v in res.values()), res
    N, D, P, k = 8192, 64, 16, 700
    Xb, Wb, ref = synth.embeddings(N, D, P, seed=17)
    ex = (np.random.default_rng(17).random(N) < 0.1).astype(np.uint8)
    X = torch.from_numpy(Xb.view(np.int16)).cuda().view(torch.bfloat16).reshape(N, D)
    W = torch.from_numpy(Wb.view(np.int16)).cuda().view(torch.bfloat16).reshape(D, P)
    idx, dd, cnt = B.select_retrain(X, W, torch.from_numpy(ref).cuda(), k, exclude=torch.from_numpy(ex).cuda())
    torch.cuda.synchronize()
    c = int(cnt.item())
    for r in range(2):
        assert np.array_equal(res[r][0], idx.cpu().numpy()[:c])
        assert np.array_equal(res[r][1], dd.cpu().numpy()[:c])
