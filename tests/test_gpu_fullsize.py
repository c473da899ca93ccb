"""Full-size parity at BASELINE.json configs[2] (ogbn-products-shaped: 2,449,029 nodes, 123.7 M
CSR entries, 100-d features, 3-layer SAGE-mean 100-256-256-47, fanout (10,25,30)) and configs[3]
(ogbn-papers100M-shaped: 111,059,956 nodes, 3.23 B CSR entries, 128-d, 2-layer 128-256-172,
fanout (10,25)), each with the memory budget bench.py calibrates so that one GPU needs >= 8
bucket groups, in the launch configuration bench.py times (bf16 feature table, tcgen05 bf16
Update GEMM).

* the plan: every seed in exactly one group, group sizes = the plan's exact block sizes,
  estimates within the budget;
* the blocks of the first and the last group: bit-exact against the oracle's C block builder
  (whole arrays: row_ptr, col_local, col_global, src_global, transposes);
* the forward: logits of sampled seeds against the oracle's forward restricted to their
  receptive field (bf16-storage reading R26, tolerance of SURVEY.md Appendix C), and the
  layer-1 Aggregate of sampled rows bit for bit (k/128 features: exact sums);
* the backward: the logits layer's bias gradient sums to zero over the classes
  (softmax - onehot rows sum to 0), and every gradient is finite.
Inputs come from synth/ only (generated on the device by synth.device, pinned bit-identical to
the numpy recipe in tests/test_synth_device.py); expected values come from oracle/ only.
"""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import CONFIGS

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, act_view, assert_bf16_close, blocks_to_numpy
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer


@pytest.fixture(scope="module", params=["products", "papers"])
def products(request):
    import bench
    cfg = CONFIGS[request.param]
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg, torch.bfloat16)
    feats = X.contiguous()
    graph = DeviceGraph(rp, col)
    kw = dict(feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    full = Trainer(graph, feats, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=1, k_max=1, **kw)
    _, _, est1, _ = full.schedule(0)
    del full
    tr = Trainer(graph, feats, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=cfg.k_min, k_max=cfg.k_max,
                 mem_budget=int(est1[0]) // 8, **kw)
    K, offs, est, ranks = tr.schedule(0)
    host = dict(rp=rp.cpu().numpy(), col=col.cpu().numpy(), y=y.cpu().numpy())

    def xrows(ids):
        """Feature rows of the given nodes, read from the synth-generated table (inputs only)."""
        idx = torch.as_tensor(np.asarray(ids, np.int64), device="cuda")
        return feats[idx, :cfg.d0].float().cpu().numpy()

    yield dict(cfg=cfg, tr=tr, K=K, offs=offs, est=est, budget=int(est1[0]) // 8, Ws=Ws, bs=bs, Xrows=xrows,
               **host, g=O.Graph(host["rp"], host["col"]))
    del tr, feats, graph, rp, col, X
    torch.cuda.empty_cache()


def test_products_plan(products):
    tr, K, offs, est = products["tr"], products["K"], products["offs"], products["est"]
    S = products["cfg"].S
    assert K >= 8 and offs[0] == 0 and offs[K] == S
    gs = tr.group_seeds.cpu().numpy()
    gos = tr.group_of_seed.cpu().numpy()                  # group of seed i, input order
    seeds = tr.seeds.cpu().numpy()
    assert np.array_equal(np.sort(gs), np.sort(seeds))    # every seed in exactly one group
    pos = np.argsort(seeds)[np.searchsorted(np.sort(seeds), gs)]
    for k in range(K):
        assert np.all(gos[pos[offs[k]:offs[k + 1]]] == k)
    assert np.all(est <= products["budget"])


@pytest.mark.slow
def test_products_plan_equals_oracle_schedule(products):
    """The full-size plan (products-shaped only: the oracle's C builder makes every item's blocks
    on the host) equals oracle.schedule run at the K the library settled on, and the same
    procedure fails at K - 1 (Alg. 3 keeps the first feasible K)."""
    if products["cfg"].N > 10_000_000:
        pytest.skip("papers100M-shaped: the host oracle would build ~60 full-size item blocks")
    tr, cfg = products["tr"], products["cfg"]
    Kt = tr.plan.k_tried
    seeds = tr.seeds.cpu().numpy()
    kw = dict(act_dtype=O.BF16, mem_budget=products["budget"], C_ppm=0)
    ref = O.schedule(products["g"], seeds, tr.L, cfg.fanout, cfg.F, tr.base_seed + 0, cfg.dims, k_min=Kt, k_max=Kt,
                     **kw)
    assert ref is not None and ref["K"] == products["K"] and ref["exploded"] == bool(tr.plan.exploded)
    np.testing.assert_array_equal(products["offs"], ref["group_offsets"])
    np.testing.assert_array_equal(products["est"], ref["est_bytes"])
    np.testing.assert_array_equal(tr.group_seeds.cpu().numpy(), ref["group_seeds"])
    if Kt > 1:
        assert O.schedule(products["g"], seeds, tr.L, cfg.fanout, cfg.F, tr.base_seed + 0, cfg.dims, k_min=Kt - 1,
                          k_max=Kt - 1, **kw) is None


def _group_blocks(products, k, seed=0):
    """Builds group k with the sampling seed of the planned epoch (seed 0): the plan's exact
    block sizes (tr.sizes_h, passed for the sync-free build) are those of that sampling."""
    tr, offs = products["tr"], products["offs"]
    L = tr.L
    n = int(offs[k + 1] - offs[k])
    tr._ensure_arena(B.estimate_mem(tr.sizes_h[k, :L + 1], tr.sizes_h[k, L + 1:], tr.model)[0])
    tr.build(int(offs[k]), n, tr.sampler(seed), tr.sizes_h[k])
    torch.cuda.synchronize()
    gseeds = tr.group_seeds[int(offs[k]):int(offs[k + 1])].cpu().numpy()
    return gseeds


@pytest.mark.parametrize("which", ["first", "last"])
def test_products_group_blocks_bit_exact(products, which):
    tr, K = products["tr"], products["K"]
    k = 0 if which == "first" else K - 1
    gseeds = _group_blocks(products, k)
    got = blocks_to_numpy(tr.arena, tr.blocks, tr.L)
    ref = O.build_blocks(products["g"], gseeds, tr.L, products["cfg"].fanout, tr.base_seed + 0)
    want_sizes = [ref[0]["n_src"]] + [b["n_dst"] for b in ref] + [b["n_edges"] for b in ref]
    np.testing.assert_array_equal(tr.sizes_h[k], want_sizes)
    for l, (a, r) in enumerate(zip(got, ref), start=1):
        for key in ("n_dst", "n_src", "n_edges"):
            assert a[key] == r[key], (l, key)
        for key in ("row_ptr", "col_local", "src_global"):
            np.testing.assert_array_equal(a[key], r[key], err_msg=f"layer {l} {key}")
        if l == 1:
            np.testing.assert_array_equal(a["col_global"], r["col_global"], err_msg="layer 1 col_global")
        else:
            np.testing.assert_array_equal(a["t_row_ptr"], r["t_row_ptr"], err_msg=f"layer {l} t_row_ptr")
            np.testing.assert_array_equal(a["t_col"], r["t_col"], err_msg=f"layer {l} t_col")


def _restricted_forward(blocks, Xrows, Ws, bs, out_rows):
    """The oracle's forward (O.mean_adjacency, O.round_bf16: bf16-storage reading R26) restricted
    to the receptive field of `out_rows` of the last block: same arithmetic as
    O.sage_forward, evaluated on the rows it needs only."""
    L = len(blocks)
    need = [None] * (L + 1)
    need[L] = np.asarray(out_rows, np.int64)
    for l in range(L, 0, -1):
        b = blocks[l - 1]
        rp, cl = b["row_ptr"].astype(np.int64), b["col_local"]
        nb = np.concatenate([cl[rp[i]:rp[i + 1]] for i in need[l]] + [need[l]])   # neighbours + self (prefix)
        need[l - 1] = np.unique(nb)
    rnd = O.round_bf16
    H = Xrows(blocks[0]["src_global"][need[0]]).astype(np.float64)
    for l in range(1, L + 1):
        b = blocks[l - 1]
        A = O.mean_adjacency(b)[need[l]][:, need[l - 1]]
        pos = np.searchsorted(need[l - 1], need[l])                  # self rows (dst i = src i)
        W = rnd(np.asarray(Ws[l - 1], np.float64))
        d_in = H.shape[1]
        agg = rnd(A @ H)
        Z = rnd(H[pos]) @ W[:, :d_in].T + agg @ W[:, d_in:].T + np.asarray(bs[l - 1], np.float64)
        H = rnd(np.maximum(Z, 0.0)) if l < L else Z
    return H


def test_products_forward_sampled(products):
    tr, cfg = products["tr"], products["cfg"]
    gseeds = _group_blocks(products, 0)
    tr.forward()
    torch.cuda.synchronize()
    ref = O.build_blocks(products["g"], gseeds, tr.L, cfg.fanout, tr.base_seed + 0)
    rng = np.random.default_rng(7)
    # layer-1 Aggregate of 4096 sampled rows: exact neighbour sums of k/128 features, then the
    # correctly rounded fp32 mean rounded to bf16 (bit for bit)
    b1 = tr.blocks.layer[0]
    rows = np.sort(rng.choice(b1.n_dst, 4096, replace=False))
    agg = act_view(tr.arena, b1.agg, b1.n_dst, b1.ld_agg, torch.bfloat16)[rows, :cfg.d0]
    A = O.mean_adjacency(ref[0])
    r0 = ref[0]
    rp = r0["row_ptr"].astype(np.int64)
    Xrows = products["Xrows"]
    nb = [r0["src_global"][r0["col_local"][rp[i]:rp[i + 1]]] for i in rows]
    flat = Xrows(np.concatenate(nb)).astype(np.float64)
    cut = np.cumsum([0] + [len(v) for v in nb])
    exact = np.stack([flat[cut[j]:cut[j + 1]].sum(0) if cut[j + 1] > cut[j] else np.zeros(cfg.d0)
                      for j in range(len(rows))])
    D = r0["D"][rows].astype(np.float32)[:, None]
    want = np.where(D > 0, exact.astype(np.float32) / np.maximum(D, 1), np.float32(0))
    want = torch.as_tensor(want).to(torch.bfloat16).float().numpy()
    np.testing.assert_array_equal(agg, want)
    assert A.shape == (r0["n_dst"], r0["n_src"])
    # logits of 24 sampled seeds against the oracle's restricted forward
    bL = tr.blocks.layer[tr.L - 1]
    srows = np.sort(rng.choice(bL.n_dst, 24, replace=False))
    logits = act_view(tr.arena, bL.out, bL.n_dst, bL.ld_out, torch.float32)[srows, :cfg.classes]
    want = _restricted_forward(ref, Xrows, products["Ws"], products["bs"], srows)
    assert_bf16_close(logits, want, "sampled logits")


def test_products_backward_properties(products):
    tr, cfg = products["tr"], products["cfg"]
    offs = products["offs"]
    tr.params.grad.zero_()
    tr.loss.zero_()
    _group_blocks(products, 0)
    tr.forward()
    tr.loss_and_grad(int(offs[0]), int(offs[1] - offs[0]))
    tr.backward()
    torch.cuda.synchronize()
    db = tr.params.db[tr.L - 1].double()
    scale = float(tr.params.db[tr.L - 1].abs().sum()) + 1e-12
    assert abs(float(db.sum())) <= 1e-3 * scale                     # sum over classes of (softmax - onehot)
    assert bool(torch.isfinite(tr.params.grad).all())
    assert float(tr.params.grad.abs().max()) > 0.0
