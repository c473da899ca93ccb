"""The pipelined epoch loop (Trainer(pipeline=True): the plan of epoch e+1 — Alg. 3, which
depends on the seeds and the epoch's sampling seed only — is computed on a side stream with its
own graph workspace while epoch e trains) gives bit-identical plans and weights to the
sequential loop (the reported loss scalar up to the order of its per-CTA float atomics)."""
import numpy as np
import pytest
import torch

from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, make_trainer


@pytest.mark.parametrize("gemm", ["ffma", "bf16"])
def test_pipelined_epochs_identical(gemm):
    N, dims, fan, F = 6000, [32, 64, 8], [5, 10], 10
    rp, col = random_graph(N, 60000, "powerlaw")
    X, y, seeds = features(N, dims[0]), labels(N, dims[-1]), seed_nodes(N, 1500)
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    mode = B.GEMM_FFMA if gemm == "ffma" else B.GEMM_BF16
    runs = []
    for pipe in (False, True):
        tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, gemm=mode, k_min=3, k_max=64, pipeline=pipe)
        hist = []
        for e in range(4):
            st = tr.run_epoch(epoch=e, lr=0.05)
            torch.cuda.synchronize()
            hist.append((st["K"], list(st["est"]), list(st["ranks"]), st["edges"], float(tr.loss.item()),
                         tr.group_seeds[: seeds.size].cpu().numpy().copy()))
        runs.append((hist, tr.params.flat.cpu().numpy().copy()))
    (h0, w0), (h1, w1) = runs
    for a, b in zip(h0, h1):
        assert a[:4] == b[:4]
        assert abs(a[4] - b[4]) <= 1e-6 * abs(a[4])     # loss: one float atomic per CTA (buffalo.h)
        np.testing.assert_array_equal(a[5], b[5])
    np.testing.assert_array_equal(w0, w1)


def test_replaced_seeds_are_scheduled_not_the_stale_plan():
    """A plan computed ahead belongs to a seed batch: set_seeds drops it, next_seeds makes the
    ahead plan for the given batch — both equal a fresh schedule of that batch."""
    N, dims, fan, F = 6000, [32, 64, 8], [5, 10], 10
    rp, col = random_graph(N, 60000, "powerlaw")
    X, y = features(N, dims[0]), labels(N, dims[-1])
    s1, s2 = seed_nodes(N, 1500), np.sort(np.random.default_rng(3).choice(N, 1500, replace=False)).astype(np.int32)
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    tr = make_trainer(rp, col, X, y, s1, dims, fan, F, Ws, bs, k_min=3, k_max=64, pipeline=True)
    ref = make_trainer(rp, col, X, y, s2, dims, fan, F, Ws, bs, k_min=3, k_max=64)
    tr.run_epoch(epoch=0, lr=0.0)                    # computes the plan of epoch 1 for s1 ahead
    tr.set_seeds(torch.as_tensor(s2).cuda())
    tr.run_epoch(epoch=1, lr=0.0, next_seeds=torch.as_tensor(s2).pin_memory())
    torch.cuda.synchronize()
    for e in (1, 2):
        if e == 2:
            tr.run_epoch(epoch=2, lr=0.0)
            torch.cuda.synchronize()
        ref.schedule(e)
        assert sorted(tr.seeds.cpu().tolist()) == sorted(s2.tolist())
        np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), ref.group_seeds.cpu().numpy())
        np.testing.assert_array_equal(tr.offs_h[: tr.plan.k_out + 1], ref.offs_h[: ref.plan.k_out + 1])
