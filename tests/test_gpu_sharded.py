"""Node-id-range sharded feature table (BASELINE.json configs[4], the IGB-shaped
configuration whose 1024-d table does not fit one GPU; the paper's data-parallel mode,
PAPER.md:458-471).

* one process, P = 3 local shards: block 1's Aggregate reads every neighbour row from its shard
  and copies the dst rows' own rows into self_rows; h_agg of layer 1 is bit-exact against the
  oracle (k/128 features: exact sums), self_rows equal the feature rows, and logits, loss and
  every gradient are bit-identical to the unsharded bf16 run (same bf16 operands in the same
  order into the same GEMMs);
* two processes sharing the GPU, each owning one shard and opening the other's over CUDA IPC
  (handles exchanged over gloo; one process per GPU on a multi-GPU box, NVLink peer loads):
  layer-1 h_agg bit-exact against the oracle and logits bit-identical to the unsharded run;
* a full-neighbour first block is refused (UNSUPPORTED).
"""
import os
import socket

import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import features, labels, random_graph, seed_nodes, xavier_weights

pytestmark = pytest.mark.gpu

N, DIMS, FAN, F = 6000, [72, 64, 48, 9], [6, 8, 10], 10


def _inputs():
    rp, col = random_graph(N, 50000, "powerlaw")
    return rp, col, features(N, DIMS[0]), labels(N, DIMS[-1]), seed_nodes(N, 1400), *xavier_weights(DIMS, bias_scale=0.05)


def _padded_bf16(X):
    from gpu_helpers import B
    pitch = B.pitch(DIMS[0])
    Xp = np.zeros((X.shape[0], pitch), np.float32)
    Xp[:, :DIMS[0]] = X[:, :DIMS[0]]
    return torch.as_tensor(Xp).cuda().to(torch.bfloat16).contiguous()


def _run(tr, seeds, seed=7):
    from gpu_helpers import B, act_view
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 16)
    tr.loss.zero_()
    tr.params.grad.zero_()
    tr.microbatch(0, seeds.size, B.make_sampler(FAN, F, seed))
    torch.cuda.synchronize()
    L = len(FAN)
    b1, bl = tr.blocks.layer[0], tr.blocks.layer[L - 1]
    agg1 = act_view(tr.arena, b1.agg, b1.n_dst, b1.ld_agg, torch.bfloat16)[:, :DIMS[0]].copy()
    logits = act_view(tr.arena, bl.out, bl.n_dst, bl.ld_out, torch.float32)[:, :DIMS[-1]].copy()
    self_rows = None
    if b1.self_rows:
        self_rows = act_view(tr.arena, b1.self_rows, b1.n_dst, b1.ld_self, torch.bfloat16)[:, :DIMS[0]].copy()
    return agg1, logits, self_rows, float(tr.loss.item()), tr.params.grad.cpu().numpy().copy()


def _expected_agg1(rp, col, X, seeds, seed=7):
    g = O.Graph(rp, col)
    blocks = O.build_blocks(g, seeds, len(FAN), FAN, seed)
    import scipy.sparse as sp
    b = blocks[0]
    A = sp.csr_matrix((np.ones(b["n_edges"]), b["col_local"], b["row_ptr"].astype(np.int64)),
                      shape=(b["n_dst"], b["n_src"]))
    S = A @ np.asarray(X[b["src_global"]][:, :DIMS[0]], np.float64)
    D = b["D"].astype(np.float32)[:, None]
    exp = np.where(D > 0, S.astype(np.float32) / np.maximum(D, 1), np.float32(0))
    return torch.as_tensor(exp).to(torch.bfloat16).float().numpy(), blocks


def test_sharded_single_process_bit_identical_to_unsharded():
    from gpu_helpers import B, make_trainer
    from paper_conf_hpca_yangzl25_b200.train import ShardedFeatures, Trainer
    rp, col, X, y, seeds, Ws, bs = _inputs()
    ref = make_trainer(rp, col, X, y, seeds, DIMS, FAN, F, Ws, bs, gemm=B.GEMM_BF16, feat_dtype=B.BF16)
    a_ref, l_ref, _, loss_ref, g_ref = _run(ref, seeds)
    table = _padded_bf16(X)
    P = 3
    rps = (N + P - 1) // P
    shards = [table[k * rps:(k + 1) * rps].clone() for k in range(P)]        # separate allocations
    feats = ShardedFeatures(shards, rps, N, table.shape[1])
    tr = Trainer((rp, col), feats, torch.as_tensor(y).cuda(), torch.as_tensor(seeds).cuda(), DIMS, FAN, F, Ws, bs,
                 feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    a, l, self_rows, loss, g = _run(tr, seeds)
    exp, blocks = _expected_agg1(rp, col, X, seeds)
    np.testing.assert_array_equal(a, exp)                                    # h_agg layer 1 vs oracle
    np.testing.assert_array_equal(a, a_ref)
    src = blocks[0]["src_global"][: blocks[0]["n_dst"]]
    np.testing.assert_array_equal(self_rows, table[torch.as_tensor(src, device="cuda").long(), :DIMS[0]].float().cpu().numpy())
    np.testing.assert_array_equal(l, l_ref)                                  # same operands, same GEMMs
    np.testing.assert_array_equal(g, g_ref)
    assert abs(loss - loss_ref) <= 1e-6 * abs(loss_ref)
    # memory model with the self-row copy: the measured arena need equals the exact model
    info_n = [tr.blocks.layer[0].n_src] + [tr.blocks.layer[l].n_dst for l in range(len(FAN))]
    info_e = [tr.blocks.layer[l].n_edges for l in range(len(FAN))]
    assert (tr.blocks.est_lo, tr.blocks.est_hi) == O.mem_model(info_n, info_e, DIMS, O.BF16, sharded=True)
    # a whole epoch through the sharded table: the plan is the oracle's with the sharded memory
    # model (its self-row copy changes M_est, so the grouping may differ from the unsharded run);
    # the accumulated gradients agree with the unsharded epoch up to the order of the groups
    tr2 = Trainer((rp, col), feats, torch.as_tensor(y).cuda(), torch.as_tensor(seeds).cuda(), DIMS, FAN, F, Ws, bs,
                  feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16, k_min=3, k_max=3)
    ref2 = make_trainer(rp, col, X, y, seeds, DIMS, FAN, F, Ws, bs, gemm=B.GEMM_BF16, feat_dtype=B.BF16, k_min=3,
                        k_max=3)
    for t in (tr2, ref2):
        t.run_epoch(epoch=1, lr=0.1)
    torch.cuda.synchronize()
    plan = O.schedule(O.Graph(rp, col), seeds, len(FAN), FAN, F, 4, DIMS, O.BF16, k_min=3, k_max=3, sharded=True)
    np.testing.assert_array_equal(tr2.group_seeds.cpu().numpy(), plan["group_seeds"])
    np.testing.assert_array_equal(tr2.offs_h[:4], plan["group_offsets"])
    # same gradients summed in another order (other groups, other split-K partials): fp32
    # summation-order differences, bounded relative to the weight scale, not to each weight
    w_ref = ref2.params.flat.cpu().numpy()
    np.testing.assert_allclose(tr2.params.flat.cpu().numpy(), w_ref, rtol=1e-5, atol=2e-5 * np.abs(w_ref).max())


def test_sharded_full_neighbour_first_block_unsupported():
    from gpu_helpers import B
    from paper_conf_hpca_yangzl25_b200.train import ShardedFeatures, Trainer
    rp, col, X, y, seeds, Ws, bs = _inputs()
    table = _padded_bf16(X)
    feats = ShardedFeatures([table], N, N, table.shape[1])
    tr = Trainer((rp, col), feats, torch.as_tensor(y).cuda(), torch.as_tensor(seeds).cuda(), DIMS, [0, 8, 10], F, Ws,
                 bs, feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    tr.group_seeds[: seeds.size].copy_(torch.as_tensor(seeds))
    tr._ensure_arena(1 << 20)
    with pytest.raises(B.BuffaloError) as ei:
        tr.build(0, seeds.size, B.make_sampler([0, 8, 10], F, 1))
    assert ei.value.status == B.ERR_UNSUPPORTED


def _ipc_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    close = None
    try:
        from gpu_helpers import B
        from paper_conf_hpca_yangzl25_b200.train import Trainer, exchange_shards
        rp, col, X, y, seeds, Ws, bs = _inputs()
        rps = (N + world - 1) // world
        table = _padded_bf16(X)
        mine = table[rank * rps:(rank + 1) * rps].clone()          # this process owns one shard
        del table
        feats, close = exchange_shards(mine, rank, world, rps, N)
        tr = Trainer((rp, col), feats, torch.as_tensor(y).cuda(), torch.as_tensor(seeds).cuda(), DIMS, FAN, F, Ws,
                     bs, feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
        a, l, _, loss, g = _run(tr, seeds)
        dist.barrier()                                              # peers done reading before close
        q.put((rank, a, l))
    finally:
        if close:
            close()
        dist.barrier()
        dist.destroy_process_group()


def test_two_processes_share_shards_over_ipc():
    import torch.multiprocessing as mp
    from gpu_helpers import B, make_trainer
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict((r, (a, l)) for r, a, l in (q.get(timeout=600) for _ in procs))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    rp, col, X, y, seeds, Ws, bs = _inputs()
    exp, _ = _expected_agg1(rp, col, X, seeds)
    ref = make_trainer(rp, col, X, y, seeds, DIMS, FAN, F, Ws, bs, gemm=B.GEMM_BF16, feat_dtype=B.BF16)
    _, l_ref, _, _, _ = _run(ref, seeds)
    for r in (0, 1):
        np.testing.assert_array_equal(res[r][0], exp)
        np.testing.assert_array_equal(res[r][1], l_ref)
