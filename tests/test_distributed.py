"""Data-parallel driver logic at world_size 2 on gloo (CPU): every rank derives the same plan
(k_min = #GPUs, LPT rank assignment, R24), runs only its own groups, and one allreduce of the
flat gradient buffer gives every rank the full-batch gradient.
Per-group gradients come from the oracle here (no GPU); the driver functions under test are
paper_conf_hpca_yangzl25_b200.train.own_groups / allreduce_grads."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights


def _setup():
    N, dims, fan, F = 400, [12, 16, 5], [3, 5], 5
    rp, col = random_graph(N, 2500, "powerlaw")
    return O.Graph(rp, col), features(N, dims[0]), labels(N, dims[-1]), seed_nodes(N, 150), dims, fan, F


def _flat(grads):
    return np.concatenate([g[0].ravel() for g in grads] + [g[1].ravel() for g in grads])


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_hpca_yangzl25_b200.train import allreduce_grads, own_groups
    g, X, y, seeds, dims, fan, F = _setup()
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    plan = O.schedule(g, seeds, 2, fan, F, 3, dims, num_gpus=world)
    mine = own_groups(plan["rank_of_group"], rank)
    acc = None
    off = plan["group_offsets"]
    for k in mine:
        sk = plan["group_seeds"][off[k]:off[k + 1]]
        _, grads, _ = O.microbatch_step(g, sk, X, y, Ws, bs, 2, fan, 3, len(seeds))
        f = _flat(grads)
        acc = f if acc is None else acc + f
    t = torch.tensor(acc if acc is not None else np.zeros_like(out[0]), dtype=torch.float64)
    allreduce_grads(t, world)
    out[rank] = t.numpy()
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_two_rank_allreduce_equals_full_batch():
    g, X, y, seeds, dims, fan, F = _setup()
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    full = O.build_blocks(g, seeds, 2, fan, 3)
    logits, cache = O.sage_forward(full, X, Ws, bs)
    _, dlog = O.softmax_ce(logits, y[seeds], len(seeds))
    ref = _flat(O.sage_backward(full, cache, Ws, dlog))
    world = 2
    mgr = mp.Manager()
    out = mgr.list([np.zeros_like(ref) for _ in range(world)])
    mp.spawn(_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    for r in range(world):
        np.testing.assert_allclose(out[r], ref, rtol=1e-10, atol=1e-13)
    # the ranks' group sets are disjoint and cover all groups
    plan = O.schedule(g, seeds, 2, fan, F, 3, dims, num_gpus=world)
    from paper_conf_hpca_yangzl25_b200.train import own_groups
    sets = [set(own_groups(plan["rank_of_group"], r)) for r in range(world)]
    assert sets[0].isdisjoint(sets[1]) and sets[0] | sets[1] == set(range(plan["K"]))
    assert plan["K"] >= world


def _ag_worker(rank, world, port, out):
    """The scheduler's all-gather callback (buffalo_sched.allgather) over gloo: called through
    its C function pointer exactly as the library calls it."""
    import ctypes
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    fn = B.make_allgather(world)
    W = 7
    send = (ctypes.c_int64 * (3 * W))(*[rank * 1000 + i for i in range(3 * W)])
    recv = (ctypes.c_int64 * (world * 3 * W))()
    cfn = ctypes.cast(fn, ctypes.c_void_p).value
    call = B.ALLGATHER_FN(cfn)
    rc = call(None, ctypes.addressof(send), ctypes.addressof(recv), 3 * W * 8)
    out[rank] = (rc, list(recv))
    dist.destroy_process_group()


def test_scheduler_allgather_callback_two_ranks():
    world = 2
    mgr = mp.Manager()
    out = mgr.list([None] * world)
    mp.spawn(_ag_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    want = [r * 1000 + i for r in range(world) for i in range(21)]
    for r in range(world):
        rc, got = out[r]
        assert rc == 0 and got == want

