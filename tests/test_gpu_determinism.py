"""include/buffalo.h promises bit-identical outputs for identical inputs and seed: two independent
runs of two epochs (fresh trainers, same synth inputs) end with bit-identical weights and plans,
for every model family and both GEMM modes."""
import numpy as np
import pytest
import torch

from synth.graphs import (features, gat_weights, labels, lstm_weights, pool_weights, random_graph, seed_nodes,
                          xavier_weights)

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, make_trainer


@pytest.mark.parametrize("model", ["mean-bf16", "mean-ffma", "pool", "lstm", "gat"])
def test_two_runs_bit_identical(model):
    N, dims, fan, F = 4000, [32, 40, 6], [4, 8], 8
    rp, col = random_graph(N, 40000, "powerlaw")
    X, y, seeds = features(N, dims[0]), labels(N, dims[-1]), seed_nodes(N, 900)
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    kw = dict(k_min=3, k_max=64)
    if model == "mean-bf16":
        kw.update(gemm=B.GEMM_BF16)
    elif model == "pool":
        Wps, bps = pool_weights(dims, bias_scale=0.05)
        kw.update(aggregator=B.AGG_POOL, Wps=Wps, bps=bps)
    elif model == "lstm":
        kw.update(aggregator=B.AGG_LSTM, lstm=lstm_weights(dims))
    elif model == "gat":
        Ws, bs, als, ars = gat_weights(dims, bias_scale=0.05)
        kw.update(aggregator=B.AGG_GAT, gat=(als, ars))
    out = []
    for _ in range(2):
        tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, pipeline=True, **kw)
        plans = []
        for e in range(2):
            st = tr.run_epoch(epoch=e, lr=0.05)
            plans.append((st["K"], list(st["est"]), st["edges"]))
        torch.cuda.synchronize()
        out.append((plans, tr.params.flat.cpu().numpy().copy()))
    assert out[0][0] == out[1][0]
    np.testing.assert_array_equal(out[0][1], out[1][1])
