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
