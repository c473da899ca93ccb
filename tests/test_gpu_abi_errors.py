"""Error behaviour of the C ABI as include/buffalo.h documents it (no exceptions across the ABI:
a status code and a message): capacity errors report the required bytes, unsupported
combinations are refused, bad arguments are rejected, and the graph workspace is restored after
a failed build so the next call still succeeds."""
import ctypes

import numpy as np
import pytest
import torch

from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B, blocks_to_numpy, make_trainer


def _trainer(**kw):
    rp, col = random_graph(2000, 12000, "powerlaw")
    dims, fan, F = [16, 24, 5], [4, 6], 6
    seeds = seed_nodes(2000, 400)
    return make_trainer(rp, col, features(2000, 16), labels(2000, 5), seeds, dims, fan, F, *xavier_weights(dims),
                        **kw), seeds, fan, F


def test_build_capacity_reports_required_and_restores_workspace():
    tr, seeds, fan, F = _trainer()
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    small = torch.empty(4096, dtype=torch.uint8, device="cuda")
    with pytest.raises(B.BuffaloError) as ei:
        B.build_blocks(tr.graph.g, tr.group_seeds.data_ptr(), seeds.size, B.make_sampler(fan, F, 1), tr.model,
                       tr.blocks, small)
    assert ei.value.status == B.ERR_CAPACITY and ei.value.required > 4096
    assert "too small" in str(ei.value)
    # the node map / bitmap were restored: a build into a big enough arena is bit-identical to a
    # build on a fresh graph workspace
    # without the plan's sizes the need is discovered while building (a lower bound per
    # attempt): grow and retry, as Trainer.build does
    size = int(ei.value.required)
    while True:
        arena = torch.empty(size, dtype=torch.uint8, device="cuda")
        try:
            B.build_blocks(tr.graph.g, tr.group_seeds.data_ptr(), seeds.size, B.make_sampler(fan, F, 1), tr.model,
                           tr.blocks, arena)
            break
        except B.BuffaloError as e:
            assert e.status == B.ERR_CAPACITY and e.required > 0
            size = max(2 * size, int(e.required * 1.25))
    a = blocks_to_numpy(arena, tr.blocks, 2)
    tr2, *_ = _trainer()
    tr2.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    arena2 = torch.empty_like(arena)
    B.build_blocks(tr2.graph.g, tr2.group_seeds.data_ptr(), seeds.size, B.make_sampler(fan, F, 1), tr2.model,
                   tr2.blocks, arena2)
    b = blocks_to_numpy(arena2, tr2.blocks, 2)
    for x, y in zip(a, b):
        for k in ("row_ptr", "col_local", "src_global"):
            np.testing.assert_array_equal(x[k], y[k])


def test_misaligned_arena_and_null_arguments():
    tr, seeds, fan, F = _trainer()
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    arena = torch.empty(1 << 24, dtype=torch.uint8, device="cuda")
    st = B.lib().buffalo_build_blocks(B.ref(tr.graph.g), tr.group_seeds.data_ptr(), seeds.size,
                                      B.ref(B.make_sampler(fan, F, 1)), B.ref(tr.model), B.ref(tr.blocks),
                                      arena.data_ptr() + 16, arena.numel() - 16, None, None,
                                      B.stream_ptr())
    assert st == B.ERR_INVALID_ARG and b"aligned" in B.lib().buffalo_last_error()
    st = B.lib().buffalo_build_blocks(B.ref(tr.graph.g), None, seeds.size, B.ref(B.make_sampler(fan, F, 1)),
                                      B.ref(tr.model), B.ref(tr.blocks), arena.data_ptr(), arena.numel(), None,
                                      None, B.stream_ptr())
    assert st == B.ERR_INVALID_ARG


def test_unsupported_combinations():
    tr, seeds, fan, F = _trainer()
    m = B.make_model([16, 24, 5], gemm_mode=B.GEMM_BF16, aggregator=B.AGG_LSTM)
    assert B.lib().buffalo_estimate_mem(2, (ctypes.c_int64 * 3)(10, 10, 10), (ctypes.c_int64 * 2)(10, 10),
                                        B.ref(m), ctypes.byref(ctypes.c_int64()),
                                        ctypes.byref(ctypes.c_int64())) == B.ERR_UNSUPPORTED
    # a mean model handed to the pool / GAT entry points
    st = B.lib().buffalo_gat_fwd(B.ref(tr.blocks.layer[0]), 1, B.ref(tr.model), 1, 16, 1, 1, 1, 1, 1, 8, 1, 1,
                                 B.stream_ptr())
    assert st == B.ERR_UNSUPPORTED
    # bf16 GEMM beyond 256 output columns
    m2 = B.make_model([16, 512, 5], gemm_mode=B.GEMM_BF16)
    assert B.lib().buffalo_estimate_mem(2, (ctypes.c_int64 * 3)(10, 10, 10), (ctypes.c_int64 * 2)(10, 10),
                                        B.ref(m2), ctypes.byref(ctypes.c_int64()),
                                        ctypes.byref(ctypes.c_int64())) == B.ERR_UNSUPPORTED


def test_clustering_workspace_capacity():
    rp, col = random_graph(1000, 5000, "powerlaw")
    g = B.Graph()
    rpt = torch.as_tensor(rp).cuda()
    colt = torch.as_tensor(col).cuda()
    g.num_nodes, g.nnz, g.row_ptr, g.col = 1000, colt.numel(), rpt.data_ptr(), colt.data_ptr()
    T = torch.empty(1000, dtype=torch.int64, device="cuda")
    ws = torch.empty(64, dtype=torch.uint8, device="cuda")
    with pytest.raises(B.BuffaloError) as ei:
        B.triangles(g, T, ws)
    assert ei.value.status == B.ERR_CAPACITY


def _graph_of(rp, col):
    g = B.Graph()
    rpt = torch.as_tensor(np.asarray(rp, np.int64)).cuda()
    colt = torch.as_tensor(np.asarray(col, np.int32)).cuda()
    g.num_nodes, g.nnz, g.row_ptr, g.col = rpt.numel() - 1, colt.numel(), rpt.data_ptr(), colt.data_ptr()
    ws = torch.empty(B.graph_workspace_bytes(g.num_nodes), dtype=torch.uint8, device="cuda")
    B.graph_prepare(g, ws)
    return g, (rpt, colt, ws)


def test_graph_validate_accepts_generator_graphs_and_names_each_violation():
    """buffalo_graph_validate checks the CSR contract of include/buffalo.h (Alg. 3 input G,
    PAPER.md:261-265): each broken rule is reported, a valid graph passes."""
    rp, col = random_graph(3000, 20000, "powerlaw")
    g, keep = _graph_of(rp, col)
    B.graph_validate(g)
    cases = {}
    c = col.copy(); r = int(np.argmax(np.diff(rp) >= 3)); c[rp[r]], c[rp[r] + 1] = c[rp[r] + 1], c[rp[r]]
    cases["not strictly increasing"] = (rp, c)
    c = col.copy(); c[rp[r] + 1] = c[rp[r]]
    cases["not strictly increasing "] = (rp, c)                   # duplicate entry
    c = col.copy(); c[-1] = 3000
    cases["outside"] = (rp, c)
    r2 = rp.copy(); r2[5], r2[6] = r2[6], r2[5]
    cases["monotone"] = (r2, col)
    c = col.copy(); v = int(np.argmax(np.diff(rp) >= 1)); c[rp[v]] = v
    cases["self loop|not strictly|symmetric"] = (rp, np.where(np.arange(c.size) == rp[v], v, col))
    for what, (r_, c_) in cases.items():
        g2, keep2 = _graph_of(r_, c_)
        with pytest.raises(B.BuffaloError) as ei:
            B.graph_validate(g2)
        assert ei.value.status == B.ERR_INVALID_ARG
        assert any(w.strip() in str(ei.value) for w in what.split("|")), (what, str(ei.value))
    # an asymmetric graph: drop one direction of one edge (rows stay sorted)
    u = int(np.argmax(np.diff(rp) >= 2))
    drop = rp[u]
    c = np.delete(col, drop)
    r_ = rp.copy(); r_[u + 1:] -= 1
    g3, keep3 = _graph_of(r_, c)
    B.graph_validate(g3, check_symmetric=False)
    with pytest.raises(B.BuffaloError) as ei:
        B.graph_validate(g3, check_symmetric=True)
    assert "symmetric" in str(ei.value)


def test_bad_seed_ids_rejected_and_plan_untouched():
    tr, seeds, fan, F = _trainer()
    pb = tr._pb[0]
    pb.offs_h[:] = -7
    pb.hist_h[:] = -7
    pb.plan.k_out = -7
    sentinel = torch.full_like(pb.group_seeds, -5)
    pb.group_seeds.copy_(sentinel)
    for bad in ("range", "negative", "duplicate"):
        s = seeds.copy()
        if bad == "range":
            s[17] = 2000
        elif bad == "negative":
            s[3] = -1
        else:
            s[100] = s[7]
        tr._seeds[0].copy_(torch.as_tensor(s))
        with pytest.raises(B.BuffaloError) as ei:
            tr.schedule(0)
        assert ei.value.status == B.ERR_INVALID_ARG
        assert ("twice" if bad == "duplicate" else "outside") in str(ei.value)
        assert pb.plan.k_out == -7 and np.all(pb.offs_h == -7) and np.all(pb.hist_h == -7)
        assert torch.equal(pb.group_seeds, sentinel)
    # the graph workspace bitmap was left clean: the valid batch schedules and builds as before
    tr._seeds[0].copy_(torch.as_tensor(seeds))
    K, offs, est, ranks = tr.schedule(0)
    assert K >= 1 and offs[-1] == seeds.size


def test_build_blocks_bad_group_ids_rejected_blocks_untouched():
    tr, seeds, fan, F = _trainer()
    arena = torch.empty(1 << 24, dtype=torch.uint8, device="cuda")
    ids = torch.as_tensor(seeds).cuda()
    B.build_blocks(tr.graph.g, ids, seeds.size, B.make_sampler(fan, F, 1), tr.model, tr.blocks, arena)
    before = bytes(tr.blocks)
    bad = ids.clone()
    bad[5] = bad[9]
    with pytest.raises(B.BuffaloError) as ei:
        B.build_blocks(tr.graph.g, bad, seeds.size, B.make_sampler(fan, F, 1), tr.model, tr.blocks, arena)
    assert ei.value.status == B.ERR_INVALID_ARG
    assert bytes(tr.blocks) == before
    small = torch.empty(4096, dtype=torch.uint8, device="cuda")
    with pytest.raises(B.BuffaloError) as ei:
        B.build_blocks(tr.graph.g, ids, seeds.size, B.make_sampler(fan, F, 1), tr.model, tr.blocks, small)
    assert ei.value.status == B.ERR_CAPACITY and bytes(tr.blocks) == before


def test_wrappers_reject_wrong_dtypes():
    tr, seeds, fan, F = _trainer()
    with pytest.raises(TypeError):
        B.bucketize(tr.graph.g, torch.as_tensor(seeds).long().cuda(), B.make_sampler(fan, F, 1), tr.model, tr.sched,
                    tr.plan, tr.bucket_ws)
    with pytest.raises(ValueError):
        B.bucketize(tr.graph.g, torch.as_tensor(seeds), B.make_sampler(fan, F, 1), tr.model, tr.sched, tr.plan,
                    tr.bucket_ws)                                          # host tensor
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 24)
    tr.build(0, seeds.size, B.make_sampler(fan, F, 1))
    b = tr.blocks.layer[0]
    with pytest.raises(TypeError):                      # fp32 model handed a bf16 feature table
        B.sage_fwd(b, 1, tr.model, tr.feats.to(torch.bfloat16), tr.feats.shape[1], tr.params.W[0], tr.params.packed[0],
                   tr.params.b[0], b.out, b.ld_out, b.agg, b.ld_agg)
    from paper_conf_hpca_yangzl25_b200.train import Trainer
    with pytest.raises(TypeError):
        Trainer(tr.graph, tr.feats, tr.labels.long(), tr.seeds, [16, 24, 5], fan, F, *xavier_weights([16, 24, 5]))
