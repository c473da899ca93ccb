"""GPU parity of GAT (Table IV; reading R30: one head per
layer) through the C ABI (buffalo_gat_fwd / buffalo_gat_bwd, driven by the Trainer) against
oracle.gat_forward / oracle.gat_backward (float64, pinned to torch.autograd on a dense masked
softmax in tests/test_oracle_gat.py).  fp32 path: SURVEY.md Appendix C tolerance (rel 1e-4,
abs 1e-5) on the attention weights, hidden activations, logits, loss and every gradient
(W, b, a_l, a_r); the arena model against the measured peak; a K = 3 epoch's plan and
accumulated gradients.  Inputs: synth/ only."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, gat_weights, labels, random_graph, seed_nodes

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, act_view, arena_view, assert_close, make_trainer

TOL = (1e-4, 1e-5)


def _case(N=2000, E=16000, S=300, fan=(5, 8), dims=(32, 24, 8), F=8):
    rp, col = random_graph(N, E, "powerlaw")
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs, als, ars = gat_weights(list(dims), bias_scale=0.05)
    return rp, col, X, y, seeds, list(fan), F, list(dims), Ws, bs, (als, ars)


@pytest.mark.parametrize("case", ["l2", "l3", "full"])
def test_gat_microbatch_parity(case):
    kw = {"l2": {}, "l3": dict(N=1500, E=9000, S=200, fan=(3, 4, 6), dims=(16, 20, 12, 5)),
          "full": dict(N=1500, E=12000, S=150, fan=(0, 6), dims=(40, 64, 7))}[case]
    rp, col, X, y, seeds, fan, F, dims, Ws, bs, att = _case(**kw)
    g = O.Graph(rp, col)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, aggregator=B.AGG_GAT, gat=att)
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    tr.loss.zero_()
    tr.params.grad.zero_()
    info = tr.microbatch(0, seeds.size, B.make_sampler(fan, F, 5))
    torch.cuda.synchronize()
    blocks = O.build_blocks(g, seeds, L, fan, 5)
    logits, cache = O.gat_forward(blocks, X, Ws, bs, *att)
    S = seeds.size
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.gat_backward(blocks, cache, Ws, att[0], att[1], dlog)
    for l in range(1, L + 1):
        bl = tr.blocks.layer[l - 1]
        # saved region: Z [n_src][pitch(d_l)], el, er, alpha [e]
        R = lambda x: (x + 255) // 256 * 256      # noqa: E731
        off = R(bl.n_src * B.pitch(dims[l]) * 4) + R(4 * bl.n_src) + R(4 * bl.n_dst)
        alpha = arena_view(tr.arena, bl.agg_saved + off, bl.n_edges, torch.float32).cpu().numpy()
        assert_close(alpha, cache[l - 1]["alpha"], *TOL, f"alpha{l}")
        if l < L:
            h = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :dims[l]]
            o = cache[l - 1]["out"]
            assert_close(h, np.where(o > 0, o, np.expm1(o)), *TOL, f"H{l}")
    bl = tr.blocks.layer[L - 1]
    glog = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :dims[-1]]
    assert_close(glog, logits, *TOL, "logits")
    assert abs(tr.loss.item() - loss) <= 1e-5 + 1e-4 * abs(loss)
    p = tr.params
    for l in range(L):
        assert_close(p.dW[l].cpu().numpy(), grads[l][0], *TOL, f"dW{l + 1}")
        assert_close(p.db[l].cpu().numpy(), grads[l][1], *TOL, f"db{l + 1}")
        assert_close(p.dal[l].cpu().numpy(), grads[l][2], *TOL, f"da_l{l + 1}")
        assert_close(p.dar[l].cpu().numpy(), grads[l][3], *TOL, f"da_r{l + 1}")
    lo, hi = O.mem_model(info["n"], info["e"], dims, O.FP32, "gat")
    assert (info["est_lo"], info["est_hi"]) == (lo, hi)
    assert lo <= info["peak"] <= hi


def test_gat_epoch_plan_and_gradients():
    rp, col, X, y, seeds, fan, F, dims, Ws, bs, att = _case(N=1500, E=12000, S=300, fan=(4, 6), dims=(24, 16, 6), F=6)
    g = O.Graph(rp, col)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, aggregator=B.AGG_GAT, gat=att,
                      k_min=3, k_max=3, base_seed=3)
    lr = 0.5
    before = tr.params.flat.clone()
    st = tr.run_epoch(epoch=0, lr=lr)
    torch.cuda.synchronize()
    applied = ((before - tr.params.flat) / lr).cpu().numpy()
    plan = O.schedule(g, seeds, L, fan, F, 3, dims, k_min=3, k_max=3, aggregator="gat")
    assert st["K"] == plan["K"]
    np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), plan["group_seeds"])
    np.testing.assert_array_equal(st["est"], plan["est_bytes"])
    off = plan["group_offsets"]
    acc, total = None, 0.0
    for k in range(plan["K"]):
        sk = plan["group_seeds"][off[k]:off[k + 1]]
        blocks = O.build_blocks(g, sk, L, fan, 3)
        lg, cache = O.gat_forward(blocks, X, Ws, bs, *att)
        loss, dlog = O.softmax_ce(lg, y[sk], seeds.size)
        gr = O.gat_backward(blocks, cache, Ws, att[0], att[1], dlog)
        total += loss
        acc = gr if acc is None else [tuple(a + b for a, b in zip(x, z)) for x, z in zip(acc, gr)]
    assert abs(tr.loss.item() - total) <= 1e-5 + 1e-4 * abs(total)
    tr.params.grad.copy_(torch.as_tensor(applied))
    p = tr.params
    for l in range(L):
        assert_close(p.dW[l].cpu().numpy(), acc[l][0], *TOL, f"dW{l + 1}")
        assert_close(p.db[l].cpu().numpy(), acc[l][1], *TOL, f"db{l + 1}")
        assert_close(p.dal[l].cpu().numpy(), acc[l][2], *TOL, f"da_l{l + 1}")
        assert_close(p.dar[l].cpu().numpy(), acc[l][3], *TOL, f"da_r{l + 1}")
