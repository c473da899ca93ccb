"""Full-size parity of the IGB-shaped configuration with a node-range sharded feature table
(BASELINE.json configs[4] at 1/8 scale, `bench.py --config igb_small`: 12.5 M nodes, 300 M CSR
entries, a 1024-d bf16 table in 8 shards of 1.56 M rows, 3-layer 1024-256-256-19, fanout
(5, 10, 15), the memory budget bench.py calibrates so that one GPU needs >= 8 bucket groups), in
the launch configuration bench.py times (sharded layer-1 Aggregate, tcgen05 bf16 Update GEMM):

* the plan: every seed in exactly one group, estimates within the budget;
* the blocks of the first group bit for bit against the oracle's C block builder;
* the layer-1 Aggregate over the shards of 4096 sampled rows bit for bit (k/128 features: exact
  sums), the dst rows' own feature rows copied to self_rows bit for bit, and the logits of
  sampled seeds against the oracle's forward restricted to their receptive field (bf16-storage
  reading R26, the Appendix C tolerance).
Inputs come from synth/ only; expected values from oracle/ only."""
import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import CONFIGS

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, act_view, assert_bf16_close, blocks_to_numpy
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, ShardedFeatures, Trainer
    from test_gpu_fullsize import _group_blocks, _restricted_forward


@pytest.fixture(scope="module")
def igb():
    import bench
    cfg = CONFIGS["igb_small"]
    P = 8
    rps = (cfg.N + P - 1) // P
    ranges = [(k * rps, min(cfg.N, (k + 1) * rps)) for k in range(P)]
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg, torch.bfloat16, ranges)
    feats = ShardedFeatures(X, rps, cfg.N, X[0].shape[1])
    graph = DeviceGraph(rp, col)
    kw = dict(feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    full = Trainer(graph, feats, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=1, k_max=1,
                   sample_cache=False, **kw)
    _, _, est1, _ = full.schedule(0)
    del full
    budget = int(est1[0]) // 8
    tr = Trainer(graph, feats, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=cfg.k_min, k_max=cfg.k_max,
                 mem_budget=budget, **kw)
    K, offs, est, ranks = tr.schedule(0)
    host = dict(rp=rp.cpu().numpy(), col=col.cpu().numpy())

    def xrows(ids):
        """Feature rows of the given nodes, read from the synth-generated shards (inputs only)."""
        ids = np.asarray(ids, np.int64)
        out = np.empty((len(ids), cfg.d0), np.float32)
        for k in range(P):
            sel = np.nonzero(ids // rps == k)[0]
            if len(sel):
                idx = torch.as_tensor(ids[sel] - k * rps, device="cuda")
                out[sel] = X[k][idx, :cfg.d0].float().cpu().numpy()
        return out

    yield dict(cfg=cfg, tr=tr, K=K, offs=offs, est=est, budget=budget, Ws=Ws, bs=bs, Xrows=xrows,
               g=O.Graph(host["rp"], host["col"]))
    del tr, feats, graph, rp, col, X
    torch.cuda.empty_cache()


def test_igb_plan(igb):
    tr, K, offs, est = igb["tr"], igb["K"], igb["offs"], igb["est"]
    S = igb["cfg"].S
    assert K >= 8 and offs[0] == 0 and offs[K] == S
    gs = tr.group_seeds.cpu().numpy()
    assert np.array_equal(np.sort(gs), np.sort(tr.seeds.cpu().numpy()))   # every seed in exactly one group
    assert np.all(est <= igb["budget"])


def test_igb_first_group_blocks_and_forward(igb):
    tr, cfg = igb["tr"], igb["cfg"]
    gseeds = _group_blocks(igb, 0)
    got = blocks_to_numpy(tr.arena, tr.blocks, tr.L)
    ref = O.build_blocks(igb["g"], gseeds, tr.L, cfg.fanout, tr.base_seed + 0)
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
    tr.forward()
    torch.cuda.synchronize()
    rng = np.random.default_rng(11)
    Xrows = igb["Xrows"]
    b1, r0 = tr.blocks.layer[0], ref[0]
    rows = np.sort(rng.choice(b1.n_dst, 4096, replace=False))
    # the dst rows' own feature rows, copied out of the shards by the Aggregate
    selfr = act_view(tr.arena, b1.self_rows, b1.n_dst, b1.ld_self, torch.bfloat16)[rows, :cfg.d0]
    np.testing.assert_array_equal(selfr, Xrows(r0["src_global"][rows]))
    # layer-1 Aggregate over the shards: exact neighbour sums of k/128 features, the correctly
    # rounded fp32 mean rounded to bf16 (bit for bit)
    agg = act_view(tr.arena, b1.agg, b1.n_dst, b1.ld_agg, torch.bfloat16)[rows, :cfg.d0]
    rp = r0["row_ptr"].astype(np.int64)
    nb = [r0["src_global"][r0["col_local"][rp[i]:rp[i + 1]]] for i in rows]
    flat = Xrows(np.concatenate(nb)).astype(np.float64)
    cut = np.cumsum([0] + [len(v) for v in nb])
    exact = np.stack([flat[cut[j]:cut[j + 1]].sum(0) if cut[j + 1] > cut[j] else np.zeros(cfg.d0)
                      for j in range(len(rows))])
    D = r0["D"][rows].astype(np.float32)[:, None]
    want = np.where(D > 0, exact.astype(np.float32) / np.maximum(D, 1), np.float32(0))
    want = torch.as_tensor(want).to(torch.bfloat16).float().numpy()
    np.testing.assert_array_equal(agg, want)
    # logits of 24 sampled seeds against the oracle's restricted forward
    bL = tr.blocks.layer[tr.L - 1]
    srows = np.sort(rng.choice(bL.n_dst, 24, replace=False))
    logits = act_view(tr.arena, bL.out, bL.n_dst, bL.ld_out, torch.float32)[srows, :cfg.classes]
    want = _restricted_forward(ref, Xrows, igb["Ws"], igb["bs"], srows)
    assert_bf16_close(logits, want, "sampled logits (sharded table)")
