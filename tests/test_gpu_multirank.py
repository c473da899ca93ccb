"""The N > 1 data-parallel path on the GPU (R24), run as 2 ranks sharing one
B200 over gloo (the sandbox has one GPU; on a multi-GPU box the same code uses NCCL, one rank per
GPU): every rank derives the same plan (k_min = #GPUs, LPT rank assignment — equal to the
oracle's), trains only its own groups with the pipelined scheduler, and one allreduce of the
flat gradient buffer gives both ranks the weights of the single-process run on the same plan
(up to the summation order of the two rank partials)."""
import os
import socket

import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

N, DIMS, FAN, F = 5000, [32, 48, 8], [5, 10], 10


def _inputs():
    rp, col = random_graph(N, 50000, "powerlaw")
    return rp, col, features(N, DIMS[0]), labels(N, DIMS[-1]), seed_nodes(N, 1200), *xavier_weights(DIMS, bias_scale=0.05)


def _train(rank, world, pg, gemm):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from gpu_helpers import B, make_trainer
    rp, col, X, y, seeds, Ws, bs = _inputs()
    mode = B.GEMM_FFMA if gemm == "ffma" else B.GEMM_BF16
    tr = make_trainer(rp, col, X, y, seeds, DIMS, FAN, F, Ws, bs, gemm=mode, k_min=2, k_max=64, rank=rank,
                      world=world, process_group=pg, pipeline=True)
    plans = []
    for e in range(3):
        st = tr.run_epoch(epoch=e, lr=0.05)
        plans.append((st["K"], list(st["ranks"]), [g["n"] for g in st["groups"]]))
    torch.cuda.synchronize()
    return tr.params.flat.cpu().numpy(), plans, tr.group_seeds.cpu().numpy()


def _worker(rank, world, port, gemm, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, *_train(rank, world, dist.group.WORLD, gemm)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("gemm", ["bf16", "ffma"])
def test_two_ranks_match_single_process(gemm):
    import torch.multiprocessing as mp
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, gemm, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict((r, (w, pl, gs)) for r, w, pl, gs in (q.get(timeout=600) for _ in procs))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    w_ref, plans_ref, gs_ref = _train(0, 1, None, gemm)
    (w0, pl0, gs0), (w1, pl1, gs1) = res[0], res[1]
    # identical plans on both ranks; the oracle's 2-GPU plan (LPT rank assignment) for epoch 0
    assert [p[:2] for p in pl0] == [p[:2] for p in pl1]
    np.testing.assert_array_equal(gs0, gs1)
    rp, col, X, y, seeds, Ws, bs = _inputs()
    ref = O.schedule(O.Graph(rp, col), seeds, 2, FAN, F, 3, DIMS, O.FP32 if gemm == "ffma" else O.BF16,
                     k_min=2, k_max=64, num_gpus=2)
    assert pl0[0][0] == ref["K"] and pl0[0][1] == list(ref["rank_of_group"])
    # each rank ran only its own groups; together all of them
    for e in range(3):
        K, ranks = pl0[e][0], pl0[e][1]
        assert len(pl0[e][2]) == sum(1 for r in ranks if r == 0) and len(pl1[e][2]) == sum(1 for r in ranks if r == 1)
        assert plans_ref[e][0] == K
    # weights: identical on both ranks (same allreduced gradients), equal to the 1-process run
    np.testing.assert_array_equal(w0, w1)
    np.testing.assert_allclose(w0, w_ref, rtol=1e-5, atol=1e-6)
