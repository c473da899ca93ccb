"""Degenerate and edge cases of the CUDA path against the oracle: a single seed, seeds without
neighbours (every seed in degree bucket 0, h_agg = 0), a fanout above every degree (blocks =
CSR slices), fanout 1, one group per seed (K = S), and a graph without edges.  Blocks and plans
bit for bit, the fp32 layer math at SURVEY.md Appendix C tolerance.  Inputs: synth/ only."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, pairs_to_csr, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, act_view, assert_close, blocks_to_numpy, make_trainer


def _graph_with_isolated(N=800, E=4000, iso=200):
    """Power-law graph on nodes [iso, N) plus `iso` isolated nodes [0, iso)."""
    rp0, col0 = random_graph(N - iso, E, "powerlaw")
    rp = np.concatenate([np.zeros(iso, np.int64), rp0]).astype(np.int64)
    col = (col0 + iso).astype(np.int32)
    return rp, col


def _check(rp, col, seeds, fan, F, dims, seed=5):
    g = O.Graph(rp, col)
    N = rp.size - 1
    X, y = features(N, dims[0]), labels(N, dims[-1])
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs)
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    tr.loss.zero_()
    tr.params.grad.zero_()
    tr.microbatch(0, seeds.size, B.make_sampler(fan, F, seed))
    torch.cuda.synchronize()
    got = blocks_to_numpy(tr.arena, tr.blocks, L)
    ref = O.build_blocks(g, seeds, L, fan, seed)
    for l, (a, r) in enumerate(zip(got, ref), start=1):
        assert (a["n_dst"], a["n_src"], a["n_edges"]) == (r["n_dst"], r["n_src"], r["n_edges"]), l
        for k in ("row_ptr", "col_local", "src_global"):
            np.testing.assert_array_equal(a[k], r[k], err_msg=f"layer {l} {k}")
    logits, cache = O.sage_forward(ref, X, Ws, bs)
    loss, dlog = O.softmax_ce(logits, y[seeds], seeds.size)
    grads = O.sage_backward(ref, cache, Ws, dlog)
    bl = tr.blocks.layer[L - 1]
    assert_close(act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :dims[-1]], logits, 1e-4, 1e-5,
                 "logits")
    for l in range(L):
        assert_close(tr.params.dW[l].cpu().numpy(), grads[l][0], 1e-4, 1e-5, f"dW{l + 1}")
        assert_close(tr.params.db[l].cpu().numpy(), grads[l][1], 1e-4, 1e-5, f"db{l + 1}")
    return tr, got, ref, g, X, y, Ws, bs


def test_single_seed():
    rp, col = random_graph(1000, 6000, "powerlaw")
    seeds = np.array([int(np.argmax(np.diff(rp)))], np.int32)         # the hub
    _check(rp, col, seeds, [4, 7], 7, [16, 24, 5])


def test_seeds_without_neighbours():
    rp, col = _graph_with_isolated()
    seeds = np.arange(0, 150, dtype=np.int32)                         # all isolated
    tr, got, ref, *_ = _check(rp, col, seeds, [3, 5], 5, [16, 24, 5])
    assert all(b["n_edges"] == 0 for b in got) and got[0]["n_src"] == seeds.size
    b = tr.blocks.layer[1]
    assert np.all(act_view(tr.arena, b.agg, b.n_dst, b.ld_agg, torch.float32) == 0.0)
    # scheduler: every seed in degree bucket 0
    g = O.Graph(rp, col)
    plan = O.schedule(g, seeds, 2, [3, 5], 5, 3, [16, 24, 5], k_min=2, k_max=2)
    assert plan["hist"][0] == seeds.size and plan["hist"][1:].sum() == 0


def test_mixed_isolated_and_connected_seeds():
    rp, col = _graph_with_isolated()
    seeds = np.sort(np.concatenate([np.arange(0, 60), np.arange(400, 520)])).astype(np.int32)
    _check(rp, col, seeds, [3, 6], 6, [16, 24, 5])


def test_fanout_above_every_degree_is_csr_slicing():
    rp, col = random_graph(600, 1500, "gnm")
    dmax = int(np.diff(rp).max())
    seeds = seed_nodes(600, 120)
    _, got, ref, *_ = _check(rp, col, seeds, [dmax + 1, dmax + 3], dmax + 3, [8, 16, 4])
    b = ref[1]
    np.testing.assert_array_equal(np.diff(b["row_ptr"]), np.diff(rp)[seeds])


def test_fanout_one():
    rp, col = random_graph(1500, 9000, "powerlaw")
    _check(rp, col, seed_nodes(1500, 300), [1, 1, 1], 1, [8, 12, 12, 4])


def test_one_group_per_seed():
    rp, col = random_graph(800, 4000, "powerlaw")
    seeds = seed_nodes(800, 24)
    dims, fan, F = [8, 16, 4], [3, 5], 5
    g = O.Graph(rp, col)
    X, y = features(800, 8), labels(800, 4)
    Ws, bs = xavier_weights(dims)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, k_min=seeds.size, k_max=seeds.size)
    K, offs, est, ranks = tr.schedule(0)
    ref = O.schedule(g, seeds, 2, fan, F, 3, dims, k_min=seeds.size, k_max=seeds.size)
    assert K == ref["K"]
    np.testing.assert_array_equal(offs, ref["group_offsets"])
    np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), ref["group_seeds"])
    np.testing.assert_array_equal(est, ref["est_bytes"])


def test_graph_without_edges():
    N = 300
    rp, col = pairs_to_csr(N, np.zeros((0, 2), np.int64))
    seeds = seed_nodes(N, 50)
    _check(np.asarray(rp, np.int64), np.asarray(col, np.int32), seeds, [2, 3], 3, [8, 16, 4])
