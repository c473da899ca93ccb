"""Pins for the oracle's GAT forward/backward (R30; Table IV).

(1) forward and every gradient (W, b, a_l, a_r) against torch.autograd on an independent dense
formulation (scores on a -inf-masked [n_dst, n_src] matrix, torch.softmax, LeakyReLU, ELU);
(2) central finite differences on a_l; (3) equal scores (a_l = a_r = 0) make the attention the
mean: out = D^-1 A Z + b."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, gat_weights, labels, random_graph, seed_nodes


def _setup(N=100, E=400, S=30, fanout=(3, 4), dims=(6, 8, 4), bias=0.1):
    rp, col = random_graph(N, E, "powerlaw")
    g = O.Graph(rp, col)
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs, als, ars = gat_weights(list(dims), bias_scale=bias)
    return g, X, y, seeds, list(fanout), list(dims), Ws, bs, als, ars


def _torch_dense(blocks, X, Ws, bs, als, ars, y_seeds, S):
    dd = torch.float64
    H = torch.tensor(np.asarray(X, np.float64)[blocks[0]["src_global"]])
    P = [[torch.tensor(np.asarray(v[l], np.float64), requires_grad=True) for l in range(len(blocks))]
         for v in (Ws, bs, als, ars)]
    L = len(blocks)
    for l in range(L):
        b = blocks[l]
        W, bb, al, ar = (P[k][l] for k in range(4))
        mask = torch.zeros(b["n_dst"], b["n_src"], dtype=torch.bool)
        for i in range(b["n_dst"]):
            mask[i, torch.tensor(b["col_local"][b["row_ptr"][i]:b["row_ptr"][i + 1]], dtype=torch.long)] = True
        Z = H @ W.T
        sc = torch.nn.functional.leaky_relu((Z @ al)[None, :] + (Z[: b["n_dst"]] @ ar)[:, None], 0.2)
        sc = torch.where(mask, sc, torch.tensor(-np.inf, dtype=dd))
        has = mask.any(1, keepdim=True)
        A = torch.where(has, torch.softmax(torch.where(has, sc, torch.zeros((), dtype=dd)), dim=1),
                        torch.zeros((), dtype=dd))
        A = torch.where(mask, A, torch.zeros((), dtype=dd))
        out = A @ Z + bb
        H = torch.nn.functional.elu(out) if l < L - 1 else out
    loss = torch.nn.functional.cross_entropy(H, torch.tensor(y_seeds, dtype=torch.long), reduction="sum") / S
    loss.backward()
    return loss.item(), H.detach().numpy(), [tuple(P[k][l].grad.numpy() for k in range(4)) for l in range(L)]


@pytest.mark.parametrize("fanout,dims", [((3, 4), (6, 8, 4)), ((2, 0, 3), (5, 6, 6, 3))])
def test_gat_matches_autograd(fanout, dims):
    g, X, y, seeds, fan, dims, Ws, bs, als, ars = _setup(fanout=fanout, dims=dims)
    L = len(fan)
    blocks = O.build_blocks(g, seeds, L, fan, 3)
    logits, cache = O.gat_forward(blocks, X, Ws, bs, als, ars)
    S = len(seeds) + 2
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.gat_backward(blocks, cache, Ws, als, ars, dlog)
    tl, tlog, tg = _torch_dense(blocks, X, Ws, bs, als, ars, y[seeds], S)
    np.testing.assert_allclose(logits, tlog, rtol=1e-12, atol=1e-12)
    assert abs(loss - tl) < 1e-12
    for ours, ref in zip(grads, tg):
        for a, r in zip(ours, ref):
            np.testing.assert_allclose(a, r, rtol=1e-9, atol=1e-12)


def test_gat_finite_differences():
    g, X, y, seeds, fan, dims, Ws, bs, als, ars = _setup(N=60, E=240, S=15, dims=(5, 6, 3))
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    S = len(seeds)

    def loss_of(als_):
        lg, _ = O.gat_forward(blocks, X, Ws, bs, als_, ars)
        return O.softmax_ce(lg, y[seeds], S)[0]

    lg, cache = O.gat_forward(blocks, X, Ws, bs, als, ars)
    _, dlog = O.softmax_ce(lg, y[seeds], S)
    grads = O.gat_backward(blocks, cache, Ws, als, ars, dlog)
    h = 1e-6
    for l in range(2):
        for k in range(len(als[l])):
            ap = [a.astype(np.float64).copy() for a in als]
            am = [a.astype(np.float64).copy() for a in als]
            ap[l][k] += h
            am[l][k] -= h
            fd = (loss_of(ap) - loss_of(am)) / (2 * h)
            assert abs(fd - grads[l][2][k]) <= 1e-7 + 1e-5 * abs(fd)


def test_gat_uniform_attention_is_mean():
    g, X, y, seeds, fan, dims, Ws, bs, als, ars = _setup()
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    zeros = [np.zeros_like(a) for a in als]
    _, cache = O.gat_forward(blocks, X, Ws, bs, zeros, zeros)
    b = blocks[0]
    A = O.mean_adjacency(b)
    want = A @ cache[0]["Z"] + np.asarray(bs[0], np.float64)
    np.testing.assert_allclose(cache[0]["out"], want, rtol=1e-13, atol=1e-14)
