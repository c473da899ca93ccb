"""Pins for the oracle's GraphSAGE-LSTM forward/backward (R29; the
paper's memory-intensive aggregator, Table III :479-497).

(1) the forward and every gradient (W, b, W_ih, W_hh, b_lstm) against torch.nn.LSTM (the library
routine, gate order i, f, g, o) run over each destination's neighbour sequence inside an autograd
graph of the whole network; (2) central finite differences on W_hh; (3) D = 1 reduces to one
LSTM cell from zero state: h = s(g_o) tanh(s(g_i) tanh(g_g)) by hand."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, lstm_weights, random_graph, seed_nodes, xavier_weights


def _setup(N=100, E=400, S=30, fanout=(3, 4), dims=(6, 8, 4), bias=0.1):
    rp, col = random_graph(N, E, "powerlaw")
    g = O.Graph(rp, col)
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs = xavier_weights(list(dims), bias_scale=bias)
    Wih, Whh, bl = lstm_weights(list(dims))
    return g, X, y, seeds, list(fanout), list(dims), Ws, bs, Wih, Whh, bl


def _torch_net(blocks, X, Ws, bs, Wih, Whh, bl, y_seeds, S):
    dd = torch.float64
    H = torch.tensor(np.asarray(X, np.float64)[blocks[0]["src_global"]])
    Wt = [torch.tensor(np.asarray(W, np.float64), requires_grad=True) for W in Ws]
    bt = [torch.tensor(np.asarray(b, np.float64), requires_grad=True) for b in bs]
    lstms = []
    L = len(blocks)
    for l in range(L):
        d = H.shape[1]
        m = torch.nn.LSTM(d, d, batch_first=True).to(dd)
        with torch.no_grad():
            m.weight_ih_l0.copy_(torch.tensor(np.asarray(Wih[l], np.float64)))
            m.weight_hh_l0.copy_(torch.tensor(np.asarray(Whh[l], np.float64)))
            m.bias_ih_l0.copy_(torch.tensor(np.asarray(bl[l], np.float64)))
            m.bias_hh_l0.zero_()
        lstms.append(m)
        b = blocks[l]
        rows = []
        for i in range(b["n_dst"]):
            nb = torch.tensor(b["col_local"][b["row_ptr"][i]:b["row_ptr"][i + 1]], dtype=torch.long)
            if len(nb) == 0:
                rows.append(torch.zeros(d, dtype=dd))
            else:
                _, (h, _) = m(H[nb][None])
                rows.append(h[0, 0])
        agg = torch.stack(rows)
        Z = H[: b["n_dst"]] @ Wt[l][:, :d].T + agg @ Wt[l][:, d:].T + bt[l]
        H = torch.relu(Z) if l < L - 1 else Z
    loss = torch.nn.functional.cross_entropy(H, torch.tensor(y_seeds, dtype=torch.long), reduction="sum") / S
    loss.backward()
    return loss.item(), H.detach().numpy(), [
        (w.grad.numpy(), b.grad.numpy(), m.weight_ih_l0.grad.numpy(), m.weight_hh_l0.grad.numpy(),
         m.bias_ih_l0.grad.numpy()) for w, b, m in zip(Wt, bt, lstms)] + \
        [np.allclose(m.bias_ih_l0.grad.numpy(), m.bias_hh_l0.grad.numpy(), rtol=1e-12, atol=1e-15) for m in lstms]


@pytest.mark.parametrize("fanout,dims", [((3, 4), (6, 8, 4)), ((2, 0, 3), (5, 6, 6, 3))])
def test_lstm_matches_torch_lstm(fanout, dims):
    g, X, y, seeds, fan, dims, Ws, bs, Wih, Whh, bl = _setup(fanout=fanout, dims=dims)
    L = len(fan)
    blocks = O.build_blocks(g, seeds, L, fan, 3)
    logits, cache = O.lstm_forward(blocks, X, Ws, bs, Wih, Whh, bl)
    S = len(seeds) + 3
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.lstm_backward(blocks, cache, Ws, Wih, Whh, dlog)
    tl, tlog, tg = _torch_net(blocks, X, Ws, bs, Wih, Whh, bl, y[seeds], S)
    tg, same_bias = tg[:L], tg[L:]
    assert all(same_bias)          # b = b_ih + b_hh: both receive the same gradient
    np.testing.assert_allclose(logits, tlog, rtol=1e-12, atol=1e-12)
    assert abs(loss - tl) < 1e-12
    for ours, ref in zip(grads, tg):
        for a, r in zip(ours, ref):
            np.testing.assert_allclose(a, r, rtol=1e-9, atol=1e-12)


def test_lstm_finite_differences():
    g, X, y, seeds, fan, dims, Ws, bs, Wih, Whh, bl = _setup(N=50, E=180, S=12, dims=(4, 5, 3))
    blocks = O.build_blocks(g, seeds, 2, fan, 3)
    S = len(seeds)

    def loss_of(Whh_):
        lg, _ = O.lstm_forward(blocks, X, Ws, bs, Wih, Whh_, bl)
        return O.softmax_ce(lg, y[seeds], S)[0]

    lg, cache = O.lstm_forward(blocks, X, Ws, bs, Wih, Whh, bl)
    _, dlog = O.softmax_ce(lg, y[seeds], S)
    grads = O.lstm_backward(blocks, cache, Ws, Wih, Whh, dlog)
    h = 1e-6
    rng = np.random.default_rng(1)
    for l in range(2):
        for _ in range(6):
            r, c = rng.integers(0, Whh[l].shape[0]), rng.integers(0, Whh[l].shape[1])
            Wp = [w.astype(np.float64).copy() for w in Whh]
            Wm = [w.astype(np.float64).copy() for w in Whh]
            Wp[l][r, c] += h
            Wm[l][r, c] -= h
            fd = (loss_of(Wp) - loss_of(Wm)) / (2 * h)
            assert abs(fd - grads[l][3][r, c]) <= 1e-7 + 1e-5 * abs(fd)


def test_lstm_single_neighbour_cell():
    g, X, y, seeds, fan, dims, Ws, bs, Wih, Whh, bl = _setup(fanout=(1, 1))
    blocks = O.build_blocks(g, seeds, 2, [1, 1], 3)
    _, cache = O.lstm_forward(blocks, X, Ws, bs, Wih, Whh, bl)
    b = blocks[0]
    H = np.asarray(X, np.float64)[b["src_global"]]
    d = H.shape[1]
    sig = lambda v: 1.0 / (1.0 + np.exp(-v))      # noqa: E731
    for i in range(b["n_dst"]):
        if b["row_ptr"][i + 1] == b["row_ptr"][i]:
            assert np.all(cache[0]["agg"][i] == 0.0)
            continue
        x = H[b["col_local"][b["row_ptr"][i]]]
        gates = np.asarray(Wih[0], np.float64) @ x + np.asarray(bl[0], np.float64)
        want = sig(gates[3 * d:]) * np.tanh(sig(gates[:d]) * np.tanh(gates[2 * d:3 * d]))
        np.testing.assert_allclose(cache[0]["agg"][i], want, rtol=1e-14, atol=1e-15)
