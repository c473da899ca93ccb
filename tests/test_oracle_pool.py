"""Pins for the oracle's GraphSAGE-pool forward/backward (R28; GraphSAGE [16] pooling
aggregator).

(1) the forward and every gradient (W, b, W_pool, b_pool) against torch.autograd on an
independent dense float64 formulation (neighbour max as amax over a -inf-masked [n_dst, n_src,
d] tensor); (2) central finite differences of the loss; (3) special cases that reduce to a
library routine: W_pool = I, b_pool = 0 and non-negative features make h_agg the element-wise
max of the neighbour rows (np.maximum.reduceat); identical rows make h_agg = ReLU(h W_pool^T +
b_pool) for every row with a neighbour; (4) the arena model's pool terms by hand."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, pool_weights, random_graph, seed_nodes, xavier_weights


def _setup(N=120, E=600, S=40, fanout=(3, 4), dims=(12, 16, 5), bias=0.1):
    rp, col = random_graph(N, E, "powerlaw")
    g = O.Graph(rp, col)
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs = xavier_weights(list(dims), bias_scale=bias)
    Wps, bps = pool_weights(list(dims), bias_scale=bias)
    return g, X, y, seeds, list(fanout), list(dims), Ws, bs, Wps, bps


def _torch_dense(blocks, X, Ws, bs, Wps, bps, y_seeds, S):
    dd = torch.float64
    H = torch.tensor(np.asarray(X, np.float64)[blocks[0]["src_global"]])
    Wt = [torch.tensor(np.asarray(W, np.float64), requires_grad=True) for W in Ws]
    bt = [torch.tensor(np.asarray(b, np.float64), requires_grad=True) for b in bs]
    Wpt = [torch.tensor(np.asarray(W, np.float64), requires_grad=True) for W in Wps]
    bpt = [torch.tensor(np.asarray(b, np.float64), requires_grad=True) for b in bps]
    L = len(blocks)
    for l in range(L):
        b = blocks[l]
        mask = torch.zeros(b["n_dst"], b["n_src"], dtype=torch.bool)
        for i in range(b["n_dst"]):
            mask[i, torch.tensor(b["col_local"][b["row_ptr"][i]:b["row_ptr"][i + 1]], dtype=torch.long)] = True
        P = torch.relu(H @ Wpt[l].T + bpt[l])                               # [n_src, d]
        big = torch.where(mask[:, :, None], P[None, :, :], torch.tensor(-np.inf, dtype=dd))
        agg = torch.amax(big, dim=1)
        agg = torch.where(mask.any(1, keepdim=True), agg, torch.zeros((), dtype=dd))
        d = H.shape[1]
        Z = H[: b["n_dst"]] @ Wt[l][:, :d].T + agg @ Wt[l][:, d:].T + bt[l]
        H = torch.relu(Z) if l < L - 1 else Z
    loss = torch.nn.functional.cross_entropy(H, torch.tensor(y_seeds, dtype=torch.long), reduction="sum") / S
    loss.backward()
    return (loss.item(), H.detach().numpy(),
            [(w.grad.numpy(), b.grad.numpy(), wp.grad.numpy(), bp.grad.numpy())
             for w, b, wp, bp in zip(Wt, bt, Wpt, bpt)])


@pytest.mark.parametrize("fanout,dims", [((3, 4), (12, 16, 5)), ((2, 0, 3), (8, 12, 12, 4))])
def test_pool_backward_matches_autograd(fanout, dims):
    g, X, y, seeds, fan, dims, Ws, bs, Wps, bps = _setup(fanout=fanout, dims=dims)
    L = len(fan)
    blocks = O.build_blocks(g, seeds, L, fan, 3)
    logits, cache = O.pool_forward(blocks, X, Ws, bs, Wps, bps)
    S = len(seeds) + 5
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.pool_backward(blocks, cache, Ws, Wps, dlog)
    tl, tlogits, tg = _torch_dense(blocks, X, Ws, bs, Wps, bps, y[seeds], S)
    np.testing.assert_allclose(logits, tlogits, rtol=1e-12, atol=1e-12)
    assert abs(loss - tl) < 1e-12
    for ours, ref in zip(grads, tg):
        for a, r in zip(ours, ref):
            np.testing.assert_allclose(a, r, rtol=1e-10, atol=1e-12)


def test_pool_finite_differences():
    g, X, y, seeds, fan, dims, Ws, bs, Wps, bps = _setup(N=60, E=240, S=15, dims=(6, 8, 3))
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    S = len(seeds)

    def loss_of(Wps_):
        lg, _ = O.pool_forward(blocks, X, Ws, bs, Wps_, bps)
        return O.softmax_ce(lg, y[seeds], S)[0]

    lg, cache = O.pool_forward(blocks, X, Ws, bs, Wps, bps)
    _, dlog = O.softmax_ce(lg, y[seeds], S)
    grads = O.pool_backward(blocks, cache, Ws, Wps, dlog)
    h = 1e-6
    rng = np.random.default_rng(0)
    for l in range(2):
        for _ in range(6):
            r, c = rng.integers(0, Wps[l].shape[0]), rng.integers(0, Wps[l].shape[1])
            Wp = [w.astype(np.float64).copy() for w in Wps]
            Wm = [w.astype(np.float64).copy() for w in Wps]
            Wp[l][r, c] += h
            Wm[l][r, c] -= h
            fd = (loss_of(Wp) - loss_of(Wm)) / (2 * h)
            assert abs(fd - grads[l][2][r, c]) <= 1e-6 + 1e-5 * abs(fd)


def test_pool_identity_transform_is_neighbour_max():
    g, X, y, seeds, fan, dims, Ws, bs, Wps, bps = _setup(dims=(12, 16, 5))
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    Xp = np.abs(X)                                        # >= 0: ReLU(I x) = x
    Wps1 = [np.eye(d, dtype=np.float32) for d in (12, 16)]
    bps0 = [np.zeros(d, np.float32) for d in (12, 16)]
    _, cache = O.pool_forward(blocks, Xp, Ws, bs, Wps1, bps0)
    b = blocks[0]
    H = Xp[b["src_global"]].astype(np.float64)
    D = np.diff(b["row_ptr"])
    nz = np.flatnonzero(D > 0)
    exp = np.maximum.reduceat(H[b["col_local"]], b["row_ptr"][:-1][nz].astype(np.int64), axis=0)
    np.testing.assert_array_equal(cache[0]["agg"][nz], exp)
    assert np.all(cache[0]["agg"][D == 0] == 0.0)
    # the recorded argmax attains the max
    arg = cache[0]["arg"]
    for i in nz[:50]:
        for k in range(12):
            if arg[i, k] >= 0:
                assert H[arg[i, k], k] == cache[0]["agg"][i, k]


def test_pool_identical_rows():
    g, X, y, seeds, fan, dims, Ws, bs, Wps, bps = _setup()
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    Xc = np.tile(X[:1], (X.shape[0], 1))
    _, cache = O.pool_forward(blocks, Xc, Ws, bs, Wps, bps)
    P1 = np.maximum(Xc[0].astype(np.float64) @ Wps[0].astype(np.float64).T + bps[0], 0.0)
    D = np.diff(blocks[0]["row_ptr"])
    np.testing.assert_allclose(cache[0]["agg"][D > 0], np.tile(P1, (int((D > 0).sum()), 1)), rtol=0, atol=1e-15)


def test_pool_memory_terms():
    n, e, dims = [1000, 300, 100], [2000, 900], [40, 64, 10]
    lo_m, hi_m = O.mem_model(n, e, dims, O.FP32, "mean")
    lo_p, hi_p = O.mem_model(n, e, dims, O.FP32, "pool")
    R = lambda x: (x + 255) // 256 * 256          # noqa: E731
    # pool adds block 1's transpose, P and argmax of both layers (activations); the backward
    # region differs by dh_agg, dQ, the pool dW/db partials and (l >= 2) no dZ/D transpose sums
    extra_persist = R(4 * 1001) + R(4 * 2000) + R(4 * 1000)
    extra_persist += R(1000 * 40 * 4) + R(300 * 40 * 4) + R(300 * 64 * 4) + R(100 * 64 * 4)
    def bwd(l, pool):
        nl, nm, din, dout = n[l], n[l - 1], dims[l - 1], dims[l]
        f = R(nl * ((dout + 7) // 8 * 8) * 4) + (R(nm * ((din + 7) // 8 * 8) * 4) if l >= 2 else 0)
        if pool:
            f += R(nl * din * 4) + R(nm * din * 4)      # dh_agg, dQ (din is a multiple of 8 here)
            S2 = O.pool_dw_splits(nm, din)
            f += R(S2 * din * din * 4) + R(S2 * din * 4)
        elif l >= 2:
            f += R(nm * ((dout + 7) // 8 * 8) * 4)
        S = O.dw_splits(nl, dout, din)
        return f + R(S * dout * 2 * din * 4) + R(S * ((dout + 7) // 8 * 8) * 4)
    blocks_m = lo_m - max(bwd(1, False), bwd(2, False))
    blocks_p = lo_p - max(bwd(1, True), bwd(2, True))
    assert blocks_p - blocks_m == extra_persist
