"""Tiny end-to-end run of every path for compute-sanitizer (tests/test_gpu_sanitizer.py):
graph validation, bucketize (K = 2), block build, forward, loss, backward and SGD for the mean
model (fp32 FFMA, bf16 tcgen05 with bf16 and fp32 feature tables), pool, LSTM and GAT, plus the
clustering coefficient.  Sizes are small so the instrumented run stays within minutes, but
large enough for several CTAs, ragged tiles and a heavy (> 128) row."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import torch  # noqa: E402

from gpu_helpers import B, make_trainer  # noqa: E402
from synth.graphs import (features, gat_weights, labels, lstm_weights, pool_weights, random_graph,  # noqa: E402
                          seed_nodes, xavier_weights)


def main(which):
    which = set(which.split(","))
    N, dims, fan, F = 1500, [24, 40, 6], [4, 0], 10
    rp, col = random_graph(N, 9000, "powerlaw")
    X, y, seeds = features(N, dims[0]), labels(N, dims[-1]), seed_nodes(N, 300)
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    runs = {
        "mean_ffma": dict(),
        "mean_bf16": dict(gemm=B.GEMM_BF16, feat_dtype=B.BF16),
        "mean_bf16_fp32feat": dict(gemm=B.GEMM_BF16),
        "pool": dict(aggregator=B.AGG_POOL, Wps=pool_weights(dims)[0], bps=pool_weights(dims)[1]),
        "lstm": dict(aggregator=B.AGG_LSTM, lstm=lstm_weights(dims)),
    }
    for name, kw in runs.items():
        if not ({"all", name} & which):
            continue
        tr = make_trainer(rp, col, X, y, seeds, dims, [4, 6] if name == "lstm" else fan, F, Ws, bs, k_min=2,
                          k_max=2, **kw)
        B.graph_validate(tr.graph.g)
        tr.run_epoch(epoch=0, lr=0.01)
        torch.cuda.synchronize()
        print(name, "ok", flush=True)
    if {"all", "gat"} & which:
        Wg, bg, als, ars = gat_weights(dims, bias_scale=0.05)
        tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Wg, bg, k_min=2, k_max=2, aggregator=B.AGG_GAT,
                          gat=(als, ars))
        tr.run_epoch(epoch=0, lr=0.01)
        torch.cuda.synchronize()
        print("gat ok", flush=True)
    if {"all", "clustering"} & which:
        T, C, ppm = B.clustering(tr.graph.g)
        torch.cuda.synchronize()
        print("clustering ok", C, flush=True)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "all")
