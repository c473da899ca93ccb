"""GPU parity of the GraphSAGE-LSTM aggregator (SURVEY §8(f) NEXT 1; PAPER.md:56, :63, :125,
:351, Table III; reading R29) through the C ABI (buffalo_lstm_fwd / buffalo_lstm_bwd, driven by
the Trainer) against oracle.lstm_forward / oracle.lstm_backward (float64, pinned to
torch.nn.LSTM in tests/test_oracle_lstm.py).  fp32 path: SURVEY.md Appendix C tolerance
(rel 1e-4, abs 1e-5) on h_agg, logits, the loss and every gradient (W, b, W_ih, W_hh, b_lstm);
the arena model (R15 with the LSTM terms) against the measured peak; a K = 3 epoch's plan
(the scheduler with the LSTM memory model) and accumulated gradients.  Inputs: synth/ only."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, lstm_weights, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, act_view, assert_close, make_trainer

TOL = (1e-4, 1e-5)


def _case(N=2000, E=16000, S=300, fan=(5, 8), dims=(32, 24, 8), F=8):
    rp, col = random_graph(N, E, "powerlaw")
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs = xavier_weights(list(dims), bias_scale=0.05)
    lstm = lstm_weights(list(dims))
    return rp, col, X, y, seeds, list(fan), F, list(dims), Ws, bs, lstm


@pytest.mark.parametrize("case", ["l2", "l3", "wide"])
def test_lstm_microbatch_parity(case):
    kw = {"l2": {}, "l3": dict(N=1500, E=9000, S=200, fan=(3, 4, 6), dims=(16, 20, 12, 5)),
          "wide": dict(N=1200, E=9000, S=150, fan=(4, 10), dims=(100, 72, 7))}[case]
    rp, col, X, y, seeds, fan, F, dims, Ws, bs, lstm = _case(**kw)
    g = O.Graph(rp, col)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, aggregator=B.AGG_LSTM, lstm=lstm)
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    tr.loss.zero_()
    tr.params.grad.zero_()
    info = tr.microbatch(0, seeds.size, B.make_sampler(fan, F, 5))
    torch.cuda.synchronize()
    blocks = O.build_blocks(g, seeds, L, fan, 5)
    logits, cache = O.lstm_forward(blocks, X, Ws, bs, *lstm)
    S = seeds.size
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.lstm_backward(blocks, cache, Ws, lstm[0], lstm[1], dlog)
    for l in range(1, L + 1):
        bl = tr.blocks.layer[l - 1]
        agg = act_view(tr.arena, bl.agg, bl.n_dst, bl.ld_agg, torch.float32)[:, :dims[l - 1]]
        assert_close(agg, cache[l - 1]["agg"], *TOL, f"h_agg{l}")
    bl = tr.blocks.layer[L - 1]
    glog = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :dims[-1]]
    assert_close(glog, logits, *TOL, "logits")
    assert abs(tr.loss.item() - loss) <= 1e-5 + 1e-4 * abs(loss)
    p = tr.params
    for l in range(L):
        assert_close(p.dW[l].cpu().numpy(), grads[l][0], *TOL, f"dW{l + 1}")
        assert_close(p.db[l].cpu().numpy(), grads[l][1], *TOL, f"db{l + 1}")
        assert_close(p.dlstm[0][l].cpu().numpy(), grads[l][2], *TOL, f"dW_ih{l + 1}")
        assert_close(p.dlstm[1][l].cpu().numpy(), grads[l][3], *TOL, f"dW_hh{l + 1}")
        assert_close(p.dlstm[2][l].cpu().numpy(), grads[l][4], *TOL, f"db_lstm{l + 1}")
    lo, hi = O.mem_model(info["n"], info["e"], dims, O.FP32, "lstm")
    assert (info["est_lo"], info["est_hi"]) == (lo, hi)
    assert lo <= info["peak"] <= hi


def test_lstm_epoch_plan_and_gradients():
    rp, col, X, y, seeds, fan, F, dims, Ws, bs, lstm = _case(N=1500, E=12000, S=300, fan=(4, 6), dims=(24, 16, 6), F=6)
    g = O.Graph(rp, col)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, aggregator=B.AGG_LSTM, lstm=lstm,
                      k_min=3, k_max=3, base_seed=3)
    lr = 0.5
    before = tr.params.flat.clone()
    st = tr.run_epoch(epoch=0, lr=lr)
    torch.cuda.synchronize()
    applied = ((before - tr.params.flat) / lr).cpu().numpy()
    plan = O.schedule(g, seeds, L, fan, F, 3, dims, k_min=3, k_max=3, aggregator="lstm")
    assert st["K"] == plan["K"]
    np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), plan["group_seeds"])
    np.testing.assert_array_equal(st["est"], plan["est_bytes"])
    off = plan["group_offsets"]
    acc, total = None, 0.0
    for k in range(plan["K"]):
        sk = plan["group_seeds"][off[k]:off[k + 1]]
        blocks = O.build_blocks(g, sk, L, fan, 3)
        lg, cache = O.lstm_forward(blocks, X, Ws, bs, *lstm)
        loss, dlog = O.softmax_ce(lg, y[sk], seeds.size)
        gr = O.lstm_backward(blocks, cache, Ws, lstm[0], lstm[1], dlog)
        total += loss
        acc = gr if acc is None else [tuple(a + b for a, b in zip(x, z)) for x, z in zip(acc, gr)]
    assert abs(tr.loss.item() - total) <= 1e-5 + 1e-4 * abs(total)
    tr.params.grad.copy_(torch.as_tensor(applied))
    p = tr.params
    for l in range(L):
        assert_close(p.dW[l].cpu().numpy(), acc[l][0], *TOL, f"dW{l + 1}")
        assert_close(p.dlstm[0][l].cpu().numpy(), acc[l][2], *TOL, f"dW_ih{l + 1}")
        assert_close(p.dlstm[1][l].cpu().numpy(), acc[l][3], *TOL, f"dW_hh{l + 1}")
        assert_close(p.dlstm[2][l].cpu().numpy(), acc[l][4], *TOL, f"db_lstm{l + 1}")


def test_lstm_rejects_long_rows():
    """A full-neighbour layer with a node of more than 128 neighbours: UNSUPPORTED (R29)."""
    rp, col, X, y, seeds, fan, F, dims, Ws, bs, lstm = _case(N=3000, E=40000, S=200, fan=(0, 4))
    assert np.diff(rp).max() > 128
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, aggregator=B.AGG_LSTM, lstm=lstm)
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    with pytest.raises(B.BuffaloError) as ei:
        tr.microbatch(0, seeds.size, B.make_sampler(fan, F, 5))
    assert ei.value.status == B.ERR_UNSUPPORTED
