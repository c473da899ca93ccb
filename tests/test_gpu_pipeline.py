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
