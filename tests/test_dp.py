"""Data-parallel retraining host logic: disjoint shards by index mod G, local
gradients scaled by 1/N_global, all-reduce sum == full-batch gradient.  CPU tests run world_size-2 gloo
process groups over the oracle; the GPU test checks the same identity on the CUDA path in-process
("virtual DP", since one box has one GPU)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from paper_conf_sigcomm_shubhas23_b200 import specs as S
from paper_conf_sigcomm_shubhas23_b200 import synth


def shard(n, rank, world):
    """a job never reuses samples other jobs use -> disjoint shards, index mod G (reading Q16)."""
    return np.arange(n)[np.arange(n) % world == rank]


def tiny():
    return {"name": "t", "in_h": 8, "in_w": 8, "in_c": 3,
            "ops": [S.conv(3, 8), S.maxpool(2, 2), S.exit_(4), S.conv(3, 8), S.exit_(4)]}


def test_shard_rule_disjoint_and_complete():
    for n in (7, 64, 1000):
        for world in (1, 2, 4, 8):
            parts = [shard(n, r, world) for r in range(world)]
            allidx = np.concatenate(parts)
            assert len(allidx) == n and len(set(allidx.tolist())) == n
            assert max(len(p) for p in parts) - min(len(p) for p in parts) <= 1


def test_virtual_dp_sum_equals_full_batch_oracle():
    spec = tiny()
    p = synth.init_params(spec, seed=1)
    xb, y = synth.drifted_images(10, 8, 8, 3, num_classes=4, seed=1)
    x = synth.bf16_bits_to_f32(xb)
    m = O.Model(spec)
    full = m.grad_exact(p.astype(np.float64), x, y, n_global=10)
    tot = np.zeros_like(full)
    for r in range(3):
        idx = shard(10, r, 3)
        tot += m.grad_exact(p.astype(np.float64), x[idx], y[idx], n_global=10)
    np.testing.assert_allclose(tot, full, rtol=1e-9, atol=1e-12)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    spec = tiny()
    p = synth.init_params(spec, seed=2)
    xb, y = synth.drifted_images(12, 8, 8, 3, num_classes=4, seed=2)
    x = synth.bf16_bits_to_f32(xb)
    idx = shard(12, rank, world)
    m = O.Model(spec)
    # one SGD step on the local shard with gradients scaled by 1/N_global, then all-reduce(sum) and update
    g = torch.from_numpy(m.grad_exact(p.astype(np.float64), x[idx], y[idx], n_global=12))
    dist.all_reduce(g, op=dist.ReduceOp.SUM)
    # replicas identical after the all-reduce (bitwise): gather a checksum
    ck = torch.tensor([float(g.sum()), float((g * g).sum())], dtype=torch.float64)
    cks = [torch.zeros_like(ck) for _ in range(world)]
    dist.all_gather(cks, ck)
    if rank == 0:
        full = m.grad_exact(p.astype(np.float64), x, y, n_global=12)
        out.put((float(np.abs(g.numpy() - full).max()), [c.tolist() for c in cks]))
    dist.destroy_process_group()


def test_gloo_world2_allreduce_equals_full_batch():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    err, cks = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert err < 1e-12
    assert cks[0] == cks[1]


@pytest.mark.gpu
def test_gpu_virtual_dp_shard_grads_sum_to_full_batch():
    """CUDA path: sum over 2 shards of retrain_step gradients (each scaled by 1/N_global) == full batch
    gradient within the 2e-2 tolerance (bf16 storage, fp32 reassociation)."""
    from paper_conf_sigcomm_shubhas23_b200 import binding as B
    from parity import rel, to_cuda_bf16
    spec = S.tiny_cnn_ee()
    p = synth.init_params(spec, seed=4)
    xb, y = synth.drifted_images(128, 32, 32, 3, seed=4)
    grads = []
    for idx in (shard(128, 0, 2), shard(128, 1, 2), np.arange(128)):
        m = B.Model(spec, 128, params=p)
        m.retrain_step(to_cuda_bf16(np.ascontiguousarray(xb[idx])), torch.from_numpy(y[idx]).cuda(), n_global=128,
                       lr=0.0)
        grads.append(m.get_grads())
        m.close()
    for kind, _i, off, shp in S.param_segments(spec):
        n = int(np.prod(shp))
        assert rel(grads[0][off:off + n] + grads[1][off:off + n], grads[2][off:off + n]) <= 2e-2, kind
