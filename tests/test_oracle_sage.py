"""Pins for the oracle's GraphSAGE-mean forward/backward and loss (Alg. 2 l.8-12).

Pins: (1) h_agg against the dense textbook formula diag(1/D) A_s H built edge by edge;
(2) mean of constant features is the constant; (3) gradients against torch.autograd on an
independent dense float64 formulation, and central finite differences; (4) the loss against
torch's cross_entropy; (5) the paper's equivalence claim:
micro-batch training is mathematically equivalent to batch training — per-seed logits of
K > 1 equal K = 1, and the accumulated partial gradients equal the full-batch gradients.
"""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights


def _setup(N=120, E=600, S=40, fanout=(3, 4), dims=(12, 16, 5), bias=0.1):
    rp, col = random_graph(N, E, "powerlaw")
    g = O.Graph(rp, col)
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs = xavier_weights(list(dims), bias_scale=bias)
    return g, X, y, seeds, list(fanout), list(dims), Ws, bs


def _dense_A(b):
    A = np.zeros((b["n_dst"], b["n_src"]))
    for i in range(b["n_dst"]):
        for e in range(b["row_ptr"][i], b["row_ptr"][i + 1]):
            A[i, b["col_local"][e]] += 1.0
    return A


def test_aggregate_matches_dense_definition():
    g, X, y, seeds, fan, dims, Ws, bs = _setup()
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    _, cache = O.sage_forward(blocks, X, Ws, bs)
    for l in range(2):
        A = _dense_A(blocks[l])
        D = A.sum(axis=1, keepdims=True)
        exp = np.where(D > 0, (A @ cache[l]["H_in"]) / np.maximum(D, 1), 0.0)
        np.testing.assert_allclose(cache[l]["agg"], exp, rtol=1e-13, atol=1e-14)


@pytest.mark.parametrize("c", [1.0, 0.5, -3.0])
def test_mean_of_constant_is_constant(c):
    g, X, y, seeds, fan, dims, Ws, bs = _setup()
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    Xc = np.full_like(X, c)
    _, cache = O.sage_forward(blocks, Xc, Ws, bs)
    agg = cache[0]["agg"]
    D = blocks[0]["D"]
    assert np.all(agg[D > 0] == c) and np.all(agg[D == 0] == 0.0)


def _torch_dense(blocks, X, Ws, bs, y_seeds, S):
    H = torch.tensor(np.asarray(X, np.float64)[blocks[0]["src_global"]])
    Wt = [torch.tensor(np.asarray(W, np.float64), requires_grad=True) for W in Ws]
    bt = [torch.tensor(np.asarray(b, np.float64), requires_grad=True) for b in bs]
    L = len(blocks)
    for l in range(L):
        A = torch.tensor(_dense_A(blocks[l]))
        D = A.sum(1, keepdim=True)
        agg = torch.where(D > 0, A @ H / D.clamp(min=1), torch.zeros(()).double())
        d = H.shape[1]
        Z = H[: blocks[l]["n_dst"]] @ Wt[l][:, :d].T + agg @ Wt[l][:, d:].T + bt[l]
        H = torch.relu(Z) if l < L - 1 else Z
    loss = torch.nn.functional.cross_entropy(H, torch.tensor(y_seeds, dtype=torch.long),
                                             reduction="sum") / S
    loss.backward()
    return loss.item(), H.detach().numpy(), [(w.grad.numpy(), b.grad.numpy()) for w, b in zip(Wt, bt)]


@pytest.mark.parametrize("fanout,dims", [((3, 4), (12, 16, 5)), ((2, 0, 3), (8, 12, 12, 4))])
def test_backward_matches_autograd(fanout, dims):
    g, X, y, seeds, fan, dims, Ws, bs = _setup(fanout=fanout, dims=dims)
    L = len(fan)
    blocks = O.build_blocks(g, seeds, L, fan, 3)
    logits, cache = O.sage_forward(blocks, X, Ws, bs)
    S = 97
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.sage_backward(blocks, cache, Ws, dlog)
    tl, tlogits, tgrads = _torch_dense(blocks, X, Ws, bs, y[seeds], S)
    np.testing.assert_allclose(logits, tlogits, rtol=1e-12, atol=1e-12)
    assert abs(loss - tl) < 1e-12
    for (gw, gb), (tw, tb) in zip(grads, tgrads):
        np.testing.assert_allclose(gw, tw, rtol=1e-10, atol=1e-13)
        np.testing.assert_allclose(gb, tb, rtol=1e-10, atol=1e-13)


def test_backward_finite_differences():
    g, X, y, seeds, fan, dims, Ws, bs = _setup(N=60, E=250, S=15)
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    Ws = [W.astype(np.float64) for W in Ws]

    def loss_of(Wl):
        logits, _ = O.sage_forward(blocks, X, Wl, bs)
        return O.softmax_ce(logits, y[seeds], 15)[0]

    logits, cache = O.sage_forward(blocks, X, Ws, bs)
    grads = O.sage_backward(blocks, cache, Ws, O.softmax_ce(logits, y[seeds], 15)[1])
    rng = np.random.default_rng(0)
    for l in range(2):
        for _ in range(5):
            i = rng.integers(Ws[l].shape[0]); j = rng.integers(Ws[l].shape[1])
            h = 1e-6
            Wp = [W.copy() for W in Ws]; Wp[l][i, j] += h
            Wm = [W.copy() for W in Ws]; Wm[l][i, j] -= h
            fd = (loss_of(Wp) - loss_of(Wm)) / (2 * h)
            assert abs(fd - grads[l][0][i, j]) < 1e-7 + 1e-5 * abs(fd)


def test_microbatch_equivalent_to_batch():
    g, X, y, seeds, fan, dims, Ws, bs = _setup(N=300, E=2000, S=120)
    full = O.build_blocks(g, seeds, 2, fan, 3)
    full_logits, cache = O.sage_forward(full, X, Ws, bs)
    _, dlog = O.softmax_ce(full_logits, y[seeds], seeds.size)
    full_grads = O.sage_backward(full, cache, Ws, dlog)
    F = fan[-1]
    plan = O.schedule(g, seeds, 2, fan, F, 3, dims, k_min=4, k_max=4)
    assert plan["K"] == 4
    acc = [(np.zeros_like(a), np.zeros_like(b)) for a, b in full_grads]
    pos = {int(s): i for i, s in enumerate(seeds)}
    off = plan["group_offsets"]
    for k in range(plan["K"]):
        sk = plan["group_seeds"][off[k]:off[k + 1]]
        blocks = O.build_blocks(g, sk, 2, fan, 3)
        logits, c = O.sage_forward(blocks, X, Ws, bs)
        np.testing.assert_allclose(logits, full_logits[[pos[int(s)] for s in sk]], rtol=0, atol=1e-12)
        _, d = O.softmax_ce(logits, y[sk], seeds.size)
        gr = O.sage_backward(blocks, c, Ws, d)
        acc = [(a + ga, b + gb) for (a, b), (ga, gb) in zip(acc, gr)]
    for (a, b), (fa, fb) in zip(acc, full_grads):
        np.testing.assert_allclose(a, fa, rtol=1e-10, atol=1e-13)
        np.testing.assert_allclose(b, fb, rtol=1e-10, atol=1e-13)


def test_train_epoch_runs_and_updates():
    g, X, y, seeds, fan, dims, Ws, bs = _setup(N=200, E=1200, S=60)
    loss, acc, newW, newb, plan = O.train_epoch(g, seeds, X, y, Ws, bs, 2, fan, fan[-1], 3, dims,
                                                lr=0.1, k_min=3, k_max=3)
    assert plan["K"] == 3 and loss > 0
    np.testing.assert_allclose(newW[0], Ws[0] - 0.1 * acc[0][0], rtol=1e-12)


def test_round_bf16_matches_torch_and_ties_to_even():
    rng = np.random.default_rng(3)
    x = np.concatenate([rng.standard_normal(10000) * 10.0 ** rng.integers(-8, 8, 10000),
                        np.array([1.0 + 2.0 ** -8, 1.0 + 3 * 2.0 ** -8, -1.0 - 2.0 ** -8, 0.0, -0.0])])
    ref = torch.as_tensor(x.astype(np.float32)).to(torch.bfloat16).double().numpy()
    np.testing.assert_array_equal(O.round_bf16(x), ref)
    # halfway cases go to the even mantissa
    assert O.round_bf16(1.0 + 2.0 ** -8) == 1.0 and O.round_bf16(1.0 + 3 * 2.0 ** -8) == 1.0 + 2.0 ** -6


def test_bf16_storage_forward_close_to_fp64():
    g, X, y, seeds, fan, dims, Ws, bs = _setup()
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    a, _ = O.sage_forward(blocks, X, Ws, bs)
    b, _ = O.sage_forward(blocks, X, Ws, bs, storage="bf16")
    assert np.linalg.norm(a - b) <= 2e-2 * np.linalg.norm(a)
    assert not np.array_equal(a, b)
