"""Measured memory high-water against the memory model (BucketMemEstimator reading R15,
PAPER.md:314, :347; the paper's Table III compares its estimate with measured memory,
PAPER.md:477-497).

The measurement is independent of the model's arithmetic and of the library's bump allocator:
the arena is filled with a sentinel word, the library is given exactly lo bytes (the model's
exact need), and after build + forward + loss + backward of a micro-batch the highest word that
no longer holds the sentinel is the high-water mark; a guard of sentinel words past lo must be
intact, and an arena of lo - 256 bytes must be refused up front.  Every model (mean fp32 / bf16,
pool, LSTM, GAT) and every group of a K = 3 plan.
"""
import numpy as np
import pytest
import torch

from synth.graphs import features, gat_weights, labels, lstm_weights, pool_weights, random_graph, seed_nodes, \
    xavier_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, make_trainer

MODELS = ["mean_ffma", "mean_bf16", "mean_bf16_fp32feat", "pool", "lstm", "gat"]


def _trainer(model):
    N, dims, fan, F = 5000, [40, 64, 48, 7], [4, 8, 12], 12
    rp, col = random_graph(N, 40000, "powerlaw")
    X, y, seeds = features(N, dims[0]), labels(N, dims[-1]), seed_nodes(N, 1200)
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    kw = dict(k_min=3, k_max=3)
    if model.startswith("mean_bf16"):
        kw.update(gemm=B.GEMM_BF16, feat_dtype=B.FP32 if model.endswith("fp32feat") else B.BF16)
    elif model == "pool":
        Wps, bps = pool_weights(dims, bias_scale=0.05)
        kw.update(aggregator=B.AGG_POOL, Wps=Wps, bps=bps)
    elif model == "lstm":
        kw.update(aggregator=B.AGG_LSTM, lstm=lstm_weights(dims))
    elif model == "gat":
        Ws, bs, als, ars = gat_weights(dims, bias_scale=0.05)
        kw.update(aggregator=B.AGG_GAT, gat=(als, ars))
    return make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, **kw)


@pytest.mark.parametrize("model", MODELS)
def test_measured_high_water_within_model(model):
    tr = _trainer(model)
    K, offs, est, ranks = tr.schedule(0)
    assert K == 3
    L = tr.L
    for k in range(K):
        hw, lo, hi, guard_ok = tr.measure_high_water(k, epoch=0)
        assert guard_ok, f"group {k}: a kernel wrote past the exact need lo = {lo}"
        assert hw <= lo <= hi
        # lo is the exact need: the backward's top slot reaches it (up to its last row's
        # 256-B padding and the unwritten padding columns of that row)
        assert lo - hw < 4096, (k, lo, hw)
        # lo - 256 bytes is refused before anything runs
        arena = torch.empty(lo - 256, dtype=torch.uint8, device="cuda")
        with pytest.raises(B.BuffaloError) as ei:
            B.build_blocks(tr.graph.g, tr.group_seeds.data_ptr() + 4 * int(offs[k]), int(offs[k + 1] - offs[k]),
                           tr.sampler(0), tr.model, tr.blocks, arena, tr.sizes_h[k])
        assert ei.value.status == B.ERR_CAPACITY and ei.value.required == lo
        # Eq. 2's estimate of the group (R = 1 here: C_ppm = 0) bounds the measured need
        assert est[k] >= hw
