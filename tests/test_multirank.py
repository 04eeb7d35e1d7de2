"""The N > 1 path on CPU: world_size-2 gloo process group.

Each rank owns the contiguous image-row shard given by the C-ABI's host-only
vista_shard_range and the whole structured table (the broadcast join).
Checked: (1) the rank-local joins partition the single-rank join exactly (pairs are
disjoint, their union is the G = 1 result); (2) the LR allreduce of per-rank partial
sums (the quantity libvista.so allreduces in fp64 over NCCL) equals the full sum.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle
from paper_conf_sigmod_nakandalak20_b200 import vista_shard_range

N, D_S, SPLIT = 240, 6, 3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, out_q):
    import torch
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    b, e = vista_shard_range(N, rank, world)
    tab = gen.make_tables(N, D_S, mismatch=True, r0=b, n_img=e - b, with_images=False)
    ps, pi, te = oracle.join(tab.img_keys, tab.str_keys, SPLIT)
    # pairs with global image rows
    pairs = np.stack([ps, pi + b, te.astype(np.int64)], 1)
    # LR partial sums over this rank's rows (structured part as features)
    X = tab.X[ps].astype(np.float64)
    y = tab.labels[ps]
    w = np.linspace(-0.2, 0.3, D_S)
    part = oracle.lr_grad_sums(X, y, te, w, 0.05)
    t = torch.from_numpy(part.copy())
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    gathered = [None] * world
    dist.all_gather_object(gathered, pairs.tolist())
    if rank == 0:
        out_q.put((t.numpy(), gathered))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_rank_join_and_allreduce():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    reduced, gathered = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # single-rank reference
    tab = gen.make_tables(N, D_S, mismatch=True, with_images=False)
    ps, pi, te = oracle.join(tab.img_keys, tab.str_keys, SPLIT)
    full = {(int(a), int(b), int(c)) for a, b, c in zip(ps, pi, te)}
    got = [tuple(p) for g in gathered for p in g]
    assert len(got) == len(set(got)) == len(full)  # disjoint shards, nothing lost
    assert set(got) == full
    X = tab.X[ps].astype(np.float64)
    w = np.linspace(-0.2, 0.3, D_S)
    ref = oracle.lr_grad_sums(X, tab.labels[ps], te, w, 0.05)
    np.testing.assert_allclose(reduced, ref, rtol=1e-12, atol=1e-12)
