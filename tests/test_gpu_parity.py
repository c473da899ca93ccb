"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded inputs.

Integer work (buckets, plan, blocks, transposes, heavy lists) must be bit-exact; fp32 (FFMA
mode) within rel 1e-4 / abs 1e-5; the bf16-GEMM path within rel 2e-2 (+ 2e-2 rms floor,
Appendix C of SURVEY.md); layer-1 aggregation of k/128 features is bit-exact in both modes.
Sizes span several tiles, ragged tails, zero-degree seeds and long-tail (heavy) rows.
"""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import (B, act_view, arena_view, assert_bf16_close, assert_close,
                             assert_normwise, blocks_to_numpy, make_trainer)


def sp_sum(b, H):
    """Exact neighbour sums of a block (float64; exact for k/128 inputs)."""
    import scipy.sparse as sp
    A = sp.csr_matrix((np.ones(b["n_edges"]), b["col_local"], b["row_ptr"].astype(np.int64)),
                      shape=(b["n_dst"], b["n_src"]))
    return A @ np.asarray(H, np.float64)

CASES = {
    # name: (N, pairs, kind, S, fanout, F, dims)
    "sampled2": (3000, 20000, "powerlaw", 700, [5, 9], 9, [40, 64, 7]),
    "full3": (4000, 30000, "powerlaw", 1500, [0, 0, 0], 10, [32, 48, 48, 10]),
    "mixed3": (5000, 60000, "powerlaw", 900, [3, 0, 25], 25, [24, 40, 56, 12]),
    "cora": (2708, 5278, "gnm", 2708, [10, 25], 25, [1433, 256, 7]),
}


def _case(name):
    N, P, kind, S, fan, F, dims = CASES[name]
    rp, col = random_graph(N, P, kind)
    X = features(N, dims[0])
    y = labels(N, dims[-1])
    seeds = seed_nodes(N, S)
    Ws, bs = xavier_weights(dims, bias_scale=0.05)
    return rp, col, X, y, seeds, fan, F, dims, Ws, bs


@pytest.mark.parametrize("name", list(CASES))
def test_blocks_bit_exact(name):
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case(name)
    g = O.Graph(rp, col)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs)
    seed = 11
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    tr.build(0, seeds.size, B.make_sampler(fan, F, seed))
    got = blocks_to_numpy(tr.arena, tr.blocks, len(fan))
    ref = O.build_blocks(g, seeds, len(fan), fan, seed)
    for l, (a, r) in enumerate(zip(got, ref), start=1):
        assert (a["n_dst"], a["n_src"], a["n_edges"]) == (r["n_dst"], r["n_src"], r["n_edges"]), l
        np.testing.assert_array_equal(a["row_ptr"], r["row_ptr"])
        np.testing.assert_array_equal(a["col_local"], r["col_local"])
        np.testing.assert_array_equal(a["src_global"], r["src_global"])
        if l == 1:
            np.testing.assert_array_equal(a["col_global"], r["col_global"])
        else:
            np.testing.assert_array_equal(a["t_row_ptr"], r["t_row_ptr"])
            np.testing.assert_array_equal(a["t_col"], r["t_col"])
        if fan[l - 1] > 0:
            # a sampled block of the mean model: natural row order, no permutation, no long rows
            assert a["cls_perm"].size == 0 and a["n_heavy"] == 0 and r["D"].max(initial=0) <= fan[l - 1]
        else:
            np.testing.assert_array_equal(a["heavy"], np.nonzero(r["D"] > O.HEAVY_T)[0])
            # degree classes (degree bucketing of the block, Alg. 2 l.6): stable sort by min(D, 129)
            cls = np.minimum(r["D"], O.HEAVY_T + 1)
            np.testing.assert_array_equal(a["cls_perm"], np.argsort(cls, kind="stable"))
        if l >= 2:
            Dt = np.diff(r["t_row_ptr"])
            np.testing.assert_array_equal(a["t_perm"], np.argsort(np.minimum(Dt, O.HEAVY_T + 1), kind="stable"))
            assert a["n_heavy_t"] == int((Dt > O.HEAVY_T).sum())
    if name == "full3":
        assert got[0]["n_heavy"] > 0          # the long-tail path is exercised


@pytest.mark.parametrize("name", list(CASES))
def test_blocks_sync_free_identical(name):
    """buffalo_build_blocks with the exact sizes given (no host round trips) builds the same
    blocks as the read-back build; the long-tail counts are then not reported."""
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case(name)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs)
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    sampler = B.make_sampler(fan, F, 11)
    tr.build(0, seeds.size, sampler)
    ref = blocks_to_numpy(tr.arena, tr.blocks, L)
    peak = tr.blocks.arena_peak
    sizes = np.array([ref[0]["n_src"]] + [b["n_dst"] for b in ref] + [b["n_edges"] for b in ref], np.int64)
    tr.arena.fill_(0xAB)
    small = tr.arena
    tr.arena = small[: peak - 256]
    with pytest.raises(B.BuffaloError) as ei:                  # capacity checked up front, exactly
        B.build_blocks(tr.graph.g, tr.group_seeds.data_ptr(), seeds.size, sampler, tr.model, tr.blocks, tr.arena,
                       sizes)
    assert ei.value.status == B.ERR_CAPACITY and ei.value.required == peak
    tr.arena = small
    B.build_blocks(tr.graph.g, tr.group_seeds.data_ptr(), seeds.size, sampler, tr.model, tr.blocks, tr.arena, sizes)
    got = blocks_to_numpy(tr.arena, tr.blocks, L)
    assert tr.blocks.arena_peak == peak
    for l, (a, r) in enumerate(zip(got, ref), start=1):
        assert a["n_heavy"] == (0 if fan[l - 1] > 0 else -1) and a["heavy"] is None and a["n_heavy_t"] == -1
        for k in ("n_dst", "n_src", "n_edges"):
            assert a[k] == r[k], (l, k)
        for k in ("row_ptr", "col_local", "src_global", "col_global", "t_row_ptr", "t_col", "cls_perm", "t_perm"):
            if r[k] is None:
                assert a[k] is None, (l, k)
            else:
                np.testing.assert_array_equal(a[k], r[k], err_msg=f"layer {l} {k}")


@pytest.mark.parametrize("name", ["sampled2", "full3", "mixed3"])
@pytest.mark.parametrize("variant", ["k4", "budget", "C", "gpus3", "gpus3_kmult"])
def test_bucketize_plan_bit_exact(name, variant):
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case(name)
    g = O.Graph(rp, col)
    kw = dict(k_min=1, k_max=4096, num_gpus=1, C_ppm=0, mem_budget=(1 << 63) - 1)
    if variant == "k4":
        kw.update(k_min=4, k_max=4)
    elif variant == "budget":
        full = O.schedule(g, seeds, len(fan), fan, F, 3, dims, k_min=1, k_max=1)
        kw.update(mem_budget=int(full["est_bytes"][0] * 0.3))
    elif variant == "C":
        full = O.schedule(g, seeds, len(fan), fan, F, 3, dims, k_min=1, k_max=1)
        kw.update(mem_budget=int(full["est_bytes"][0] * 0.3), C_ppm=226000)
    elif variant == "gpus3":
        kw.update(num_gpus=3)
    else:                                       # R31: rank-aware K (multiples of #GPUs) under a budget
        full = O.schedule(g, seeds, len(fan), fan, F, 3, dims, k_min=1, k_max=1)
        kw.update(num_gpus=3, k_multiple=3, mem_budget=int(full["est_bytes"][0] * 0.2))
    ref = O.schedule(g, seeds, len(fan), fan, F, 3, dims, **kw)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, base_seed=3,
                      **{k: v for k, v in kw.items() if k != "num_gpus"}, world=kw["num_gpus"])
    if variant == "gpus3_kmult":
        assert ref["K_tried"] % 3 == 0
    K, offs, est, ranks = tr.schedule(0)
    assert K == ref["K"] and tr.plan.k_tried == ref["K_tried"]
    assert bool(tr.plan.exploded) == ref["exploded"] and tr.plan.num_items == ref["num_items"]
    np.testing.assert_array_equal(offs, ref["group_offsets"])
    np.testing.assert_array_equal(est, ref["est_bytes"])
    np.testing.assert_array_equal(ranks, ref["rank_of_group"])
    np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), ref["group_seeds"])
    np.testing.assert_array_equal(tr.group_of_seed.cpu().numpy(), ref["group_of_seed"])
    np.testing.assert_array_equal(tr.hist_h, ref["hist"])
    # exact block sizes of this rank's groups (plan.group_sizes_h) = the oracle's blocks of that
    # group; the rows of other ranks' groups are -1 (each rank measures its own)
    L = len(fan)
    gs = ref["group_seeds"]
    for k in range(K):
        if kw["num_gpus"] > 1 and ranks[k] != 0:
            assert np.all(tr.sizes_h[k] == -1)
            continue
        blocks = O.build_blocks(g, gs[offs[k]:offs[k + 1]], L, fan, 3)
        want = [blocks[0]["n_src"]] + [b["n_dst"] for b in blocks] + [b["n_edges"] for b in blocks]
        np.testing.assert_array_equal(tr.sizes_h[k], want, err_msg=f"group {k}")


def test_bucketize_random_instances_vs_plain_loop():
    """The library's K loop (with the R25 fast paths and batched micro-bucket statistics)
    against the oracle's plain Alg. 3 loop (fast_paths=False) on random instances: K, the
    explosion flag (R7) and the whole plan bit for bit."""
    rng = np.random.default_rng(77)
    rp, col = random_graph(2000, 12000, "powerlaw")
    g = O.Graph(rp, col)
    n_exp = 0
    for it in range(24):
        S = int(rng.integers(50, 1500))
        seeds = np.sort(rng.choice(g.N, S, replace=False)).astype(np.int32)
        L = int(rng.integers(1, 4))
        fan = [int(rng.choice([0, 3, 5, 10])) for _ in range(L)]
        F = int(rng.integers(2, 11)) if fan[-1] <= 0 else fan[-1]
        dims = [int(rng.integers(4, 48)) for _ in range(L + 1)]
        full = O.schedule(g, seeds, L, fan, F, 3, dims, k_min=1, k_max=1)
        budget = int(full["est_bytes"][0] * rng.uniform(0.1, 1.0))
        gpus = int(rng.choice([1, 2, 3]))
        ref = O.schedule(g, seeds, L, fan, F, 3, dims, mem_budget=budget, k_max=40, num_gpus=gpus,
                         fast_paths=False)
        X = np.zeros((g.N, dims[0]), np.float32)
        y = np.zeros(g.N, np.int32)
        Ws, bs = xavier_weights(dims)
        tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, base_seed=3, mem_budget=budget, k_max=40,
                          world=gpus)
        if ref is None:
            with pytest.raises(B.BuffaloError) as ei:
                tr.schedule(0)
            assert ei.value.status == B.ERR_BUDGET
            continue
        K, offs, est, ranks = tr.schedule(0)
        n_exp += ref["exploded"]
        assert (K, tr.plan.k_tried, bool(tr.plan.exploded)) == (ref["K"], ref["K_tried"], ref["exploded"]), it
        np.testing.assert_array_equal(offs, ref["group_offsets"])
        np.testing.assert_array_equal(est, ref["est_bytes"])
        np.testing.assert_array_equal(ranks, ref["rank_of_group"])
        np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), ref["group_seeds"])
    assert n_exp >= 3


def test_bucketize_budget_error():
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case("sampled2")
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, mem_budget=4096, k_max=16)
    with pytest.raises(B.BuffaloError) as ei:
        tr.schedule(0)
    assert ei.value.status == B.ERR_BUDGET


def _run_microbatch(tr, seeds, fan, F, seed):
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    tr.loss.zero_()
    tr.params.grad.zero_()
    info = tr.microbatch(0, seeds.size, B.make_sampler(fan, F, seed))
    torch.cuda.synchronize()
    return info


@pytest.mark.parametrize("name", list(CASES))
@pytest.mark.parametrize("gemm", ["ffma", "bf16", "bf16feat"])
def test_microbatch_fwd_bwd_parity(name, gemm):
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case(name)
    g = O.Graph(rp, col)
    L = len(fan)
    mode = B.GEMM_FFMA if gemm == "ffma" else B.GEMM_BF16
    fdt = B.BF16 if gemm == "bf16feat" else B.FP32      # bf16 feature table: the bench's configuration
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, gemm=mode, feat_dtype=fdt)
    S = seeds.size
    info = _run_microbatch(tr, seeds, fan, F, 7)
    blocks = O.build_blocks(g, seeds, L, fan, 7)
    logits, cache = O.sage_forward(blocks, X, Ws, bs, "fp64" if mode == B.GEMM_FFMA else "bf16")
    loss, dlog = O.softmax_ce(logits, y[seeds], S)
    grads = O.sage_backward(blocks, cache, Ws, dlog)
    adt = torch.float32 if mode == B.GEMM_FFMA else torch.bfloat16
    # layer-1 aggregation of k/128 features: the neighbour sums are exact in fp32, so h_agg is
    # the correctly rounded fp32 quotient (then rounded to bf16 in the bf16 mode), bit for bit
    b1 = tr.blocks.layer[0]
    agg1 = act_view(tr.arena, b1.agg, b1.n_dst, b1.ld_agg, adt)[:, :dims[0]]
    rb = blocks[0]
    S_exact = sp_sum(rb, X[rb["src_global"]])
    D = rb["D"].astype(np.float32)[:, None]
    exp = np.where(D > 0, S_exact.astype(np.float32) / np.maximum(D, 1), np.float32(0))
    if mode == B.GEMM_BF16:
        exp = torch.as_tensor(exp).to(torch.bfloat16).float().numpy()
    np.testing.assert_array_equal(agg1, exp)
    bl = tr.blocks.layer[L - 1]
    glog = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :dims[-1]]
    gW = [w.cpu().numpy() for w in tr.params.dW]
    gb = [b.cpu().numpy() for b in tr.params.db]
    if mode == B.GEMM_FFMA:
        assert_close(glog, logits, 1e-4, 1e-5, "logits")
        assert abs(tr.loss.item() - loss) <= 1e-5 + 1e-4 * abs(loss)
        for l in range(L):
            assert_close(gW[l], grads[l][0], 1e-4, 1e-5, f"dW{l + 1}")
            assert_close(gb[l], grads[l][1], 1e-4, 1e-5, f"db{l + 1}")
    else:
        assert_bf16_close(glog, logits, "logits")
        assert abs(tr.loss.item() - loss) <= 2e-2 * abs(loss)
        for l in range(L):
            assert_bf16_close(gW[l], grads[l][0], f"dW{l + 1}")
            assert_bf16_close(gb[l], grads[l][1], f"db{l + 1}")
    # memory model: the measured arena peak lies in [lo, hi] and equals the oracle's model
    lo, hi = O.mem_model(info["n"], info["e"], dims, O.FP32 if mode == B.GEMM_FFMA else O.BF16)
    assert (info["est_lo"], info["est_hi"]) == (lo, hi)
    assert lo <= info["peak"] <= hi


@pytest.mark.parametrize("name", list(CASES))
def test_bf16_layer_outputs_vs_plain_fp64(name):
    """bf16 mode against the PLAIN float64 oracle (no bf16 rounding anywhere in the reference),
    layer by layer and fed the same inputs: for each layer l the reference takes the GPU's own
    layer input H_{l-1} (the feature table at l = 1) and computes h_agg = D^-1 A H_{l-1} and
    Z_l = [H_self || h_agg] W_l^T + b_l in float64 with the fp32 master weights; the GPU's H_l
    (= ReLU(Z_l) stored in bf16) and logits must match elementwise within the north star's
    rel 2e-2 (+ 2e-2 rms floor).  Feeding each layer the GPU's input keeps
    near-zero pre-activations of earlier layers from compounding (R26)."""
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case(name)
    g = O.Graph(rp, col)
    L = len(fan)
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, gemm=B.GEMM_BF16, feat_dtype=B.BF16)
    _run_microbatch(tr, seeds, fan, F, 7)
    blocks = O.build_blocks(g, seeds, L, fan, 7)
    H = np.asarray(X, np.float64)[blocks[0]["src_global"]][:, :dims[0]]
    for l in range(1, L + 1):
        b = tr.blocks.layer[l - 1]
        A = O.mean_adjacency(blocks[l - 1])
        agg = A @ H
        W = np.asarray(Ws[l - 1], np.float64)
        d_in = dims[l - 1]
        Z = H[: b.n_dst] @ W[:, :d_in].T + agg @ W[:, d_in:].T + np.asarray(bs[l - 1], np.float64)
        if l < L:
            got = act_view(tr.arena, b.out, b.n_dst, b.ld_out, torch.bfloat16)[:, :dims[l]]
            assert_bf16_close(got, np.maximum(Z, 0.0), f"H_{l} vs plain fp64")
            H = got.astype(np.float64)                 # the GPU's layer input for the next layer
        else:
            got = act_view(tr.arena, b.out, b.n_dst, b.ld_out, torch.float32)[:, :dims[l]]
            assert_bf16_close(got, Z, "logits vs plain fp64")


@pytest.mark.parametrize("name", ["sampled2", "mixed3"])
def test_ffma_general_fp32_features(name):
    """FFMA mode on Gaussian fp32 features (not the k/128 grid, so fp32 sums round and their
    order matters) against the float64 oracle at rel 1e-4 / abs 1e-5: h_agg of every layer,
    logits, loss and all gradients."""
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case(name)
    g = O.Graph(rp, col)
    L = len(fan)
    Xg = np.random.default_rng(5).standard_normal(X.shape).astype(np.float32)
    tr = make_trainer(rp, col, Xg, y, seeds, dims, fan, F, Ws, bs)
    _run_microbatch(tr, seeds, fan, F, 7)
    blocks = O.build_blocks(g, seeds, L, fan, 7)
    logits, cache = O.sage_forward(blocks, Xg, Ws, bs)
    loss, dlog = O.softmax_ce(logits, y[seeds], seeds.size)
    grads = O.sage_backward(blocks, cache, Ws, dlog)
    H = np.asarray(Xg, np.float64)[blocks[0]["src_global"]][:, :dims[0]]
    for l in range(1, L + 1):
        b = tr.blocks.layer[l - 1]
        agg = act_view(tr.arena, b.agg, b.n_dst, b.ld_agg, torch.float32)[:, :dims[l - 1]]
        ref_agg = O.mean_adjacency(blocks[l - 1]) @ H
        assert_close(agg, ref_agg, 1e-4, 1e-5, f"h_agg layer {l}")
        if l < L:
            H = act_view(tr.arena, b.out, b.n_dst, b.ld_out, torch.float32)[:, :dims[l]].astype(np.float64)
    bl = tr.blocks.layer[L - 1]
    assert_close(act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :dims[-1]], logits, 1e-4, 1e-5,
                 "logits")
    assert abs(tr.loss.item() - loss) <= 1e-5 + 1e-4 * abs(loss)
    for l in range(L):
        assert_close(tr.params.dW[l].cpu().numpy(), grads[l][0], 1e-4, 1e-5, f"dW{l + 1}")
        assert_close(tr.params.db[l].cpu().numpy(), grads[l][1], 1e-4, 1e-5, f"db{l + 1}")


def test_mean_of_constant_is_constant():
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case("full3")
    Xc = np.full_like(X, 0.5)
    tr = make_trainer(rp, col, Xc, y, seeds, dims, fan, F, Ws, bs)
    _run_microbatch(tr, seeds, fan, F, 1)
    b1 = tr.blocks.layer[0]
    agg = act_view(tr.arena, b1.agg, b1.n_dst, b1.ld_agg, torch.float32)[:, :dims[0]]
    D = np.diff(arena_view(tr.arena, b1.row_ptr, b1.n_dst + 1).cpu().numpy())
    assert np.all(agg[D > 0] == 0.5) and np.all(agg[D == 0] == 0.0)


@pytest.mark.parametrize("gemm", ["ffma", "bf16", "bf16feat"])
def test_microbatch_logits_equal_batch_logits(gemm):
    """micro-batch training is equivalent to batch training; on the GPU the
    per-seed logits of a group equal the full batch's bit for bit (row-local reductions)."""
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case("mixed3")
    mode = B.GEMM_FFMA if gemm == "ffma" else B.GEMM_BF16
    fdt = B.BF16 if gemm == "bf16feat" else B.FP32
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, gemm=mode, feat_dtype=fdt)
    _run_microbatch(tr, seeds, fan, F, 5)
    bl = tr.blocks.layer[-1 + len(fan)]
    full = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32).copy()
    pos = {int(s): i for i, s in enumerate(seeds)}
    for part in np.array_split(seeds[::-1].copy(), 3):
        _run_microbatch(tr, part, fan, F, 5)
        bl = tr.blocks.layer[len(fan) - 1]
        sub = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)
        np.testing.assert_array_equal(sub, full[[pos[int(s)] for s in part]])


@pytest.mark.parametrize("gemm", ["ffma", "bf16", "bf16feat"])
def test_epoch_parity(gemm):
    """Alg. 2 end to end: plan, accumulated gradients over K = 4 groups, one SGD step."""
    rp, col, X, y, seeds, fan, F, dims, Ws, bs = _case("sampled2")
    g = O.Graph(rp, col)
    mode = B.GEMM_FFMA if gemm == "ffma" else B.GEMM_BF16
    fdt = B.BF16 if gemm == "bf16feat" else B.FP32
    tr = make_trainer(rp, col, X, y, seeds, dims, fan, F, Ws, bs, gemm=mode, k_min=4, k_max=4, base_seed=3,
                      feat_dtype=fdt)
    lr = 0.5
    stats = tr.run_epoch(epoch=2, lr=lr)
    torch.cuda.synchronize()
    loss, acc, newW, newb, plan = O.train_epoch(g, seeds, X, y, Ws, bs, len(fan), fan, F, 5, dims, lr=lr,
                                                storage="fp64" if mode == B.GEMM_FFMA else "bf16",
                                                k_min=4, k_max=4)
    assert stats["K"] == plan["K"] == 4
    for l in range(len(fan)):
        if mode == B.GEMM_FFMA:
            assert_close(tr.params.W[l].cpu().numpy(), newW[l], 1e-4, 1e-5, f"W{l + 1}")
            assert_close(tr.params.b[l].cpu().numpy(), newb[l], 1e-4, 1e-5, f"b{l + 1}")
        else:
            assert_bf16_close(tr.params.W[l].cpu().numpy() - Ws[l], newW[l] - Ws[l], f"dW{l + 1}")
    assert float(tr.params.grad.abs().max()) == 0.0       # gradients reset by the step
