"""Full-size forward parity of the widened models: GraphSAGE-pool and GAT
on the ogbn-products-shaped graph of BASELINE.json configs[2] (2.45 M nodes, 123.7 M CSR
entries, 100-256-256-47, fanout (10,25,30)) and GraphSAGE-LSTM on the paper's arxiv LSTM workload
(`arxiv_lstm`), in the fp32 launch configuration bench.py times for them.

The first group of the plan is built and run forward on the GPU; the oracle's C builder makes the
same group's blocks, which are cut down to the receptive field of 24 sampled seeds (sub-blocks
keep each row's neighbours in CSR order and the dst-prefix-of-src layout), and the oracle's own
pool_forward / gat_forward / lstm_forward run on them.  Logits compared at SURVEY.md Appendix C's
fp32 tolerance (the forward uses maxima and softmaxes, which are continuous in their inputs).
Inputs: synth/ only."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import CONFIGS, gat_weights, lstm_weights, pool_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, act_view, assert_close
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer


def _sub_blocks(blocks, rows):
    """The blocks restricted to the receptive field of dst rows `rows` of the last block."""
    L = len(blocks)
    subs = [None] * L
    order = np.asarray(rows, np.int64)                     # dst order of sub-block L
    for l in range(L, 0, -1):
        b = blocks[l - 1]
        rp = b["row_ptr"].astype(np.int64)
        cl = b["col_local"]
        nbr = [cl[rp[i]:rp[i + 1]] for i in order]
        in_dst = np.zeros(b["n_src"], bool)
        in_dst[order] = True
        rest = np.unique(np.concatenate(nbr + [np.zeros(0, np.int32)]).astype(np.int64))
        rest = rest[~in_dst[rest]]
        src = np.concatenate([order, rest])                # dst prefix, then the other sources
        pos = np.full(b["n_src"], -1, np.int64)
        pos[src] = np.arange(src.size)
        D = np.array([len(x) for x in nbr], np.int64)
        subs[l - 1] = dict(n_dst=order.size, n_src=src.size, n_edges=int(D.sum()),
                           row_ptr=np.concatenate([[0], np.cumsum(D)]).astype(np.int32),
                           col_local=(pos[np.concatenate(nbr)] if D.sum() else np.zeros(0, np.int64)).astype(np.int32),
                           src_global=b["src_global"][src], D=D.astype(np.int32))
        order = src
    return subs


def _run(cfg_name, aggregator, kw, oracle_fwd, k_min=8):
    import bench
    cfg = CONFIGS[cfg_name]
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg)
    if aggregator == B.AGG_GAT:
        Ws, bs, als, ars = gat_weights(cfg.dims)
        kw = dict(gat=(als, ars))
    graph = DeviceGraph(rp, col)
    tr = Trainer(graph, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, gemm_mode=B.GEMM_FFMA, k_min=k_min,
                 k_max=max(k_min, 64), aggregator=aggregator, **kw)
    K, offs, est, ranks = tr.schedule(0)
    n = int(offs[1] - offs[0])
    L = tr.L
    tr._ensure_arena(B.estimate_mem(tr.sizes_h[0, :L + 1], tr.sizes_h[0, L + 1:], tr.model)[0])
    tr.build(0, n, tr.sampler(0), tr.sizes_h[0])
    tr.forward()
    torch.cuda.synchronize()
    bL = tr.blocks.layer[L - 1]
    rng = np.random.default_rng(3)
    rows = np.sort(rng.choice(bL.n_dst, 24, replace=False))
    got = act_view(tr.arena, bL.out, bL.n_dst, bL.ld_out, torch.float32)[rows, :cfg.classes]
    gseeds = tr.group_seeds[:n].cpu().numpy()
    g = O.Graph(rp.cpu().numpy(), col.cpu().numpy())
    blocks = O.build_blocks(g, gseeds, L, cfg.fanout, tr.base_seed + 0)
    subs = _sub_blocks(blocks, rows)
    # the oracle indexes X by src_global of block 1: pass only the rows it needs
    need = subs[0]["src_global"]
    Xs = X[torch.as_tensor(need.astype(np.int64), device=X.device), :cfg.d0].double().cpu().numpy()
    subs[0] = dict(subs[0], src_global=np.arange(need.size))
    want, _ = oracle_fwd(subs, Xs, Ws, bs)
    return got, want


def test_pool_products_sampled_logits():
    cfg = CONFIGS["products"]
    Wps, bps = pool_weights(cfg.dims)
    got, want = _run("products", B.AGG_POOL, dict(Wps=Wps, bps=bps),
                     lambda s, X, W, b: O.pool_forward(s, X, W, b, Wps, bps))
    assert_close(got, want, 1e-4, 1e-5, "pool logits (products-shaped)")


def test_gat_products_sampled_logits():
    cfg = CONFIGS["products"]
    _, _, als, ars = gat_weights(cfg.dims)
    got, want = _run("products", B.AGG_GAT, {}, lambda s, X, W, b: O.gat_forward(s, X, W, b, als, ars))
    assert_close(got, want, 1e-4, 1e-5, "GAT logits (products-shaped)")


def test_lstm_arxiv_sampled_logits():
    cfg = CONFIGS["arxiv_lstm"]
    lw = lstm_weights(cfg.dims)
    got, want = _run("arxiv_lstm", B.AGG_LSTM, dict(lstm=lw), lambda s, X, W, b: O.lstm_forward(s, X, W, b, *lw),
                     k_min=2)
    assert_close(got, want, 1e-4, 1e-5, "LSTM logits (arxiv LSTM workload)")
