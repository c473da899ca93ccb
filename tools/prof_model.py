"""Profiling driver (diagnostic): one epoch of a widened model (pool / gat / lstm / mean-ffma) on
a products-shaped graph (arxiv-shaped for lstm), for ncu launch lists filtered to the library's
kernels.  Not a benchmark (bench.py is)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from synth.graphs import CONFIGS, gat_weights, lstm_weights, pool_weights  # noqa: E402


def main():
    agg = sys.argv[1] if len(sys.argv) > 1 else "pool"
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import Trainer
    cfg = CONFIGS["arxiv_lstm" if agg == "lstm" else "products"]
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg)
    kw = dict(feat_dtype=B.FP32, gemm_mode=B.GEMM_FFMA)
    if agg == "pool":
        Wps, bps = pool_weights(cfg.dims)
        kw.update(aggregator=B.AGG_POOL, Wps=Wps, bps=bps)
    elif agg == "gat":
        Ws, bs, als, ars = gat_weights(cfg.dims)
        kw.update(aggregator=B.AGG_GAT, gat=(als, ars))
    elif agg == "lstm":
        kw.update(aggregator=B.AGG_LSTM, lstm=lstm_weights(cfg.dims))
    tr = Trainer((rp, col), X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=8 if agg != "lstm" else 3,
                 k_max=8 if agg != "lstm" else 3, **kw)
    tr.run_epoch(epoch=0, lr=0.0)
    torch.cuda.synchronize()
    print("K", tr.last["K"])


if __name__ == "__main__":
    main()
