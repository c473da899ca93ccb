"""Buffalo CPU ORACLE (test infrastructure only; see oracle/__init__.py).

A plain, slow, obviously-correct restatement of what Buffalo's hot path computes, written
from /root/reference/PAPER.md (cited as PAPER.md:<line>) and the readings listed in
DESIGN.md §"Readings of the paper" (cited as R<n>).  Integer work (sampling, blocks) is in
oracle/buffalo_oracle.c (plain C, single thread); the scheduler is plain Python; the layer
math is numpy/scipy in float64.  Nothing here is shared with the CUDA path.

Functions and the passages they follow:
  degree_bucketing     Alg. 3 l.1, PAPER.md:127 ("nodes with a larger degree than F are
                       grouped together into a single bucket"), :164, :269; R1, R5
  item_stats           Eq. 1 inputs I, O, D "obtained during the micro-batch generation"
                       PAPER.md:386; R13
  mem_model            BucketMemEstimator PAPER.md:314/:347 — delegated by the paper to
                       Betty [93]; our reading R15 = exact arena bytes of one micro-batch
  grouping_weight      Eq. 1 + Eq. 2, PAPER.md:359-363 (integer form, R14)
  split_explosion      SplitExplosionBucket PAPER.md:273, :335 ("evenly splits"); R7, R8
  mem_balanced_group   Alg. 4 PAPER.md:313-326 with text :343 (largest first, R10)
  schedule             Alg. 3 PAPER.md:269-280 + :333 (K loop, K=1 special case)
  build_blocks         Alg. 2 l.5 PAPER.md:237 + §IV-E :388-390 (C); transposes by definition
  sage_forward         Alg. 2 l.8-9 PAPER.md:240-241 (Aggregate = mean, Update = W_l) with
                       GraphSAGE-mean [16]; R20, R21; bf16-storage variant R26
  round_bf16           IEEE round-to-nearest-even to bfloat16 (R26)
  softmax_ce           Alg. 2 l.10 PAPER.md:242; normalisation by the global batch (R19)
  sage_backward        Alg. 2 l.11-12 PAPER.md:243-244 (gradients accumulated over groups)
  train_epoch          Alg. 2 PAPER.md:233-245 end to end (one optimizer step, R18)
  pool_forward, pool_backward
                       GraphSAGE-pool (the paper's aggregators "mean, pool
                       or LSTM", "Our method is general and applicable to any
                       aggregators", :386; pool as defined by GraphSAGE [16]): P = ReLU(H W_pool^T
                       + b_pool), h_agg = element-wise max over the sampled neighbours, then the
                       same Update as mean (R28)
  lstm_forward, lstm_backward
                       GraphSAGE-LSTM (the paper's memory-intensive
                       aggregator, Table III :479-497): an LSTM with
                       hidden size d_{l-1} run over each destination's sampled neighbours in CSR
                       order, h_agg = its last hidden state (R29)
  gat_forward, gat_backward
                       GAT (the paper's second model, Table IV
                       :499-513; GAT [68]/[32]) on the same blocks: one attention head per layer,
                       LeakyReLU(0.2) scores, softmax over the sampled neighbours, ELU between
                       layers (R30)
  triangles, avg_clustering
                       C of Eq. 1 (Newman's local clustering
                       coefficient, "page 142 of reference [27]"): T_v by definition (C),
                       C = mean over all nodes of 2 T_v / (d_v (d_v - 1)), 0 for d_v < 2 (R27)
"""
import ctypes
import math
import os
import subprocess

import numpy as np
import scipy.sparse as sp

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "buffalo_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

INT64_MAX = (1 << 63) - 1


# ============================================================================ C library
def build_lib(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


class _OBlock(ctypes.Structure):
    _fields_ = [("n_dst", ctypes.c_int64), ("n_src", ctypes.c_int64), ("n_edges", ctypes.c_int64),
                ("row_ptr", ctypes.POINTER(ctypes.c_int32)),
                ("col_local", ctypes.POINTER(ctypes.c_int32)),
                ("col_global", ctypes.POINTER(ctypes.c_int32)),
                ("src_global", ctypes.POINTER(ctypes.c_int32))]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build_lib())
        P = ctypes.c_void_p
        _lib.oracle_philox.argtypes = [P, P, P]
        _lib.oracle_sample_row.argtypes = [P, P, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64,
                                           ctypes.c_int32, P]
        _lib.oracle_sample_row.restype = ctypes.c_int64
        _lib.oracle_build_blocks.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int64,
                                             ctypes.c_int32, P, ctypes.c_uint64, P]
        _lib.oracle_build_blocks.restype = ctypes.c_int
        _lib.oracle_triangles.argtypes = [P, P, ctypes.c_int64, ctypes.c_int64, P]
        _lib.oracle_triangles.restype = None
        _lib.oracle_block_sizes.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int64,
                                            ctypes.c_int32, P, ctypes.c_uint64, P, P]
        _lib.oracle_block_sizes.restype = ctypes.c_int
        _lib.oracle_free_blocks.argtypes = [P, ctypes.c_int32]
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


class Graph:
    """CSR graph: row_ptr int64[N+1], col int32[nnz] (rows sorted, no duplicates)."""

    def __init__(self, row_ptr, col):
        self.row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
        self.col = np.ascontiguousarray(col, dtype=np.int32)
        self.N = self.row_ptr.size - 1

    def degree(self, v):
        return self.row_ptr[np.asarray(v, dtype=np.int64) + 1] - self.row_ptr[np.asarray(v, dtype=np.int64)]


def philox(ctr, key):
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().oracle_philox(_p(c), _p(k), _p(out))
    return out


def sample_row(g, v, f, seed, hop):
    out = np.zeros(max(1, int(g.degree(v))), dtype=np.int32)
    n = lib().oracle_sample_row(_p(g.row_ptr), _p(g.col), int(v), int(f), int(seed), int(hop), _p(out))
    return out[:n].copy()


# ============================================================================ blocks
def build_blocks(g, seeds, L, fanout, seed):
    """Blocks l = 1..L (returned as a list indexed l-1) of the micro-batch with output nodes
    `seeds` (Alg. 2 l.5).  Each block is a dict with
    n_dst, n_src, n_edges, row_ptr, col_local, col_global, src_global, D (= row lengths) and
    the transposed block t_row_ptr / t_col (for each src j, the dst i with an edge to j,
    ascending i)."""
    seeds = np.ascontiguousarray(seeds, dtype=np.int32)
    fan = np.ascontiguousarray(fanout, dtype=np.int32)
    arr = (_OBlock * L)()
    rc = lib().oracle_build_blocks(g.N, _p(g.row_ptr), _p(g.col), _p(seeds), seeds.size, L, _p(fan),
                                   int(seed), ctypes.cast(arr, ctypes.c_void_p))
    if rc != 0:
        raise MemoryError("oracle_build_blocks failed")
    blocks = []
    for l in range(1, L + 1):
        b = arr[l - 1]
        nd, ns, ne = b.n_dst, b.n_src, b.n_edges
        rp = np.ctypeslib.as_array(b.row_ptr, shape=(nd + 1,)).copy()
        cl = np.ctypeslib.as_array(b.col_local, shape=(max(ne, 1),))[:ne].copy()
        cg = np.ctypeslib.as_array(b.col_global, shape=(max(ne, 1),))[:ne].copy()
        sg = np.ctypeslib.as_array(b.src_global, shape=(max(ns, 1),))[:ns].copy()
        D = np.diff(rp).astype(np.int64)
        dst_of_edge = np.repeat(np.arange(nd, dtype=np.int32), D)
        order = np.argsort(cl, kind="stable")
        t_col = dst_of_edge[order].astype(np.int32)
        t_rp = np.zeros(ns + 1, dtype=np.int32)
        np.cumsum(np.bincount(cl, minlength=ns), out=t_rp[1:])
        blocks.append(dict(n_dst=nd, n_src=ns, n_edges=ne, row_ptr=rp, col_local=cl,
                           col_global=cg, src_global=sg, D=D, t_row_ptr=t_rp, t_col=t_col))
    lib().oracle_free_blocks(ctypes.cast(arr, ctypes.c_void_p), L)
    return blocks


def block_sizes(g, seeds, L, fanout, seed):
    """(n[0..L], e[1..L] as a list indexed l-1) of the blocks of `seeds`."""
    seeds = np.ascontiguousarray(seeds, dtype=np.int32)
    fan = np.ascontiguousarray(fanout, dtype=np.int32)
    n = np.zeros(L + 1, dtype=np.int64)
    e = np.zeros(L, dtype=np.int64)
    rc = lib().oracle_block_sizes(g.N, _p(g.row_ptr), _p(g.col), _p(seeds), seeds.size, L,
                                  _p(fan), int(seed), _p(n), _p(e))
    if rc != 0:
        raise MemoryError("oracle_block_sizes failed")
    return [int(x) for x in n], [int(x) for x in e]


# ============================================================================ bucketing
def degree_bucketing(g, seeds, f_L, F):
    """Alg. 3 l.1 DegreeBucketing.  D(v) = min(deg(v), f_L) (deg(v) for
    a full-neighbour output layer, f_L <= 0); bucket(v) = min(D(v), F); the degree-F bucket
    holds every node with D >= F.  Returns (D, bucket, order, hist): `order` lists seed
    positions grouped by bucket ascending, input order inside a bucket (R5)."""
    seeds = np.asarray(seeds, dtype=np.int64)
    deg = g.degree(seeds)
    D = deg if f_L <= 0 else np.minimum(deg, f_L)
    bucket = np.minimum(D, F)
    order = np.argsort(bucket, kind="stable")
    hist = np.bincount(bucket, minlength=F + 1)
    return D.astype(np.int64), bucket.astype(np.int64), order.astype(np.int64), hist.astype(np.int64)


# ============================================================================ memory model
ALIGN = 256
HEAVY_T = 128          # rows with D > HEAVY_T go through the cooperative long-tail path
FP32, BF16 = 0, 1
SCAN_TILE = 4096       # elements per tile of the implementation's device-wide scans
PART_TILE = 4096       # elements per tile of its stable radix/bin partition passes
DB_SPLITS = 296        # row splits of the bf16 path's deterministic db reduction
BWD_DB_PARTS = 148 * 5 + 148   # db partial rows of the bf16 backward's fused transposed Aggregate


def _R(x):
    return ((int(x) + ALIGN - 1) // ALIGN) * ALIGN


def _ceil(a, b):
    return (int(a) + int(b) - 1) // int(b)


def pitch(d):
    return ((int(d) + 7) // 8) * 8


def dw_splits(n_l, d_out, d_in):
    """Split count of the deterministic split-K dW reduction."""
    tiles = _ceil(d_out, 64) * _ceil(2 * d_in, 64)
    return max(1, min(_ceil(592, tiles), _ceil(n_l, 512)))


def tc_dw_splits(n_l, d_out, d_in):
    """Split count of the tensor-core dW reduction (one CTA per 256-column tile of [2 Dp] and
    row split, all of d_out per CTA)."""
    Dp = _ceil(d_in, 64) * 64
    tiles = _ceil(2 * Dp, 256)
    return max(1, min(_ceil(148, tiles), _ceil(max(int(n_l), 1), 512)))


def _part_count_elems(e):
    return 256 * _ceil(max(int(e), 1), PART_TILE)


def _scan_ws_bytes(length):
    return _R(8 * (_ceil(max(int(length), 1), SCAN_TILE) + 2))


def pool_dw_splits(n_rows, d):
    """Split count of the pool weight's dW reduction (K = d columns, d rows)."""
    tiles = _ceil(d, 64) * _ceil(d, 64)
    return max(1, min(_ceil(592, tiles), _ceil(n_rows, 512)))


def gemm_splits(n_rows, rows_out, K):
    """Split count of a deterministic split-K reduction over n_rows (rows_out x K result)."""
    tiles = _ceil(rows_out, 64) * _ceil(K, 64)
    return max(1, min(_ceil(592, tiles), _ceil(max(int(n_rows), 1), 512)))


def lstm_dw_splits(n_rows, d):
    """Split count of the LSTM weights' dW reduction (4d rows, K = d columns)."""
    tiles = _ceil(4 * d, 64) * _ceil(d, 64)
    return max(1, min(_ceil(592, tiles), _ceil(max(int(n_rows), 1), 512)))


def mem_model(n, e, dims, act_dtype=FP32, aggregator="mean", sharded=False):
    """BucketMemEstimator reading R15: the exact arena bytes of one
    micro-batch with layer sizes n[0..L], e[1..L] (e indexed l-1) and widths dims[0..L].
    Returns (lo, hi): hi = capacity that always suffices (used as M_est), lo = bytes the
    backward pass is certain to touch; the measured arena peak lies in [lo, hi].
    Every buffer is rounded up to 256 B.  Restated from DESIGN.md §5 "Arena".  sharded: the
    feature table is sharded over processes, so block 1 keeps a bf16 copy of its
    dst rows' feature rows (the Update / dW operand)."""
    L = len(e)
    s = 4 if act_dtype == FP32 else 2
    pool = aggregator == "pool"                  # R28: fp32 only; block 1 keeps a transpose too
    lstm = aggregator == "lstm"                  # R29: fp32 only
    gat = aggregator == "gat"                    # R30: fp32 only; block 1 keeps a transpose too
    blocks = 0
    build = 0
    for l in range(1, L + 1):
        nl, nm, el = n[l], n[l - 1], e[l - 1]
        blocks += _R(4 * (nl + 1)) + _R(4 * nl) + _R(4 * el) + _R(4 * nm)   # row_ptr cls_perm col src
        if l == 1:
            blocks += _R(4 * el)                                # col_global kept for layer 1
            if pool or gat:
                blocks += _R(4 * (nm + 1)) + _R(4 * el) + _R(4 * nm)
        else:
            blocks += _R(4 * (nm + 1)) + _R(4 * el) + _R(4 * nm)  # transposed block + its classes
        pne = _part_count_elems(nl + el)
        frame = _R(64) + _scan_ws_bytes(max(nl + el + 1, pne + 1))
        frame += _R(4 * (pne + 1))                              # partition counts (classes, radix)
        if l >= 2:
            frame += _R(4 * el) + _R(4 * (nl + el))             # col_global + transpose cursors
        elif pool or gat:
            frame += _R(4 * (nl + el))                          # transpose cursors of block 1
        build = max(build, frame)
    acts = 0
    for l in range(1, L + 1):
        if not gat:
            acts += _R(n[l] * pitch(dims[l - 1]) * s)           # saved h_agg
        if l < L:
            acts += _R(n[l] * pitch(dims[l]) * s)               # H_l
    acts += _R(n[L] * pitch(dims[L]) * 4)                       # logits
    if sharded:
        acts += _R(n[1] * pitch(dims[0]) * 2)                   # block 1's self-row copy (bf16)
    if gat:
        for l in range(1, L + 1):                               # Z, el, er, alpha per edge
            acts += _R(n[l - 1] * pitch(dims[l]) * 4) + _R(4 * n[l - 1]) + _R(4 * n[l]) + _R(4 * e[l - 1])
    if lstm:
        for l in range(1, L + 1):
            d, el, nl = dims[l - 1], e[l - 1], n[l]
            acts += _R(el * pitch(4 * d) * 4)                   # gates (i, f, u, o), later their gradients
            acts += _R(el * pitch(d) * 4)                       # cell state c_t per (dst, step)
            acts += 2 * _R(el * 4)                              # source row and packed position per edge
            acts += 2 * _R(nl * pitch(d) * 4)                   # running h, c (backward: dh, dc)
            acts += _R(4 * 256)                                 # degree-class counts, max degree
    if pool:
        for l in range(1, L + 1):
            acts += _R(n[l - 1] * pitch(dims[l - 1]) * 4)       # P = ReLU(H W_pool^T + b_pool)
            acts += _R(n[l] * pitch(dims[l - 1]) * 4)           # argmax (local src index)

    def dh_slot(l):                                             # dH_l slot of the backward region
        if act_dtype == BF16 and l < L:                         # bf16 dZ_l + its db partial rows
            return _R(n[l] * pitch(dims[l]) * 2) + _R(4 * BWD_DB_PARTS * dims[l])
        return _R(n[l] * pitch(dims[l]) * 4)                    # fp32 dH / dlogits

    bwd = 0
    for l in range(L, 0, -1):
        frame = dh_slot(l)
        if l >= 2:
            frame += dh_slot(l - 1)
        if pool:
            d = dims[l - 1]
            frame += _R(n[l] * pitch(d) * 4) + _R(n[l - 1] * pitch(d) * 4)     # dh_agg, dQ
            S2 = pool_dw_splits(n[l - 1], d)
            frame += _R(S2 * d * d * 4) + _R(S2 * pitch(d) * 4)               # dW_pool, db_pool partials
        if gat:
            din, dl, ns, nd, el = dims[l - 1], dims[l], n[l - 1], n[l], e[l - 1]
            frame += _R(ns * pitch(dl) * 4) + _R(4 * el) + _R(4 * ns) + _R(4 * nd)   # dZ, ds, d_el, d_er
            S4, Sl, Sr = gemm_splits(ns, dl, din), gemm_splits(ns, 1, dl), gemm_splits(nd, 1, dl)
            frame += _R(S4 * dl * din * 4) + _R(S4 * pitch(dl) * 4)                 # dW partials
            frame += _R(Sl * dl * 4) + _R(Sl * 4) + _R(Sr * dl * 4) + _R(Sr * 4)     # da_l, da_r partials
            bwd = max(bwd, frame)
            continue
        if lstm:
            d, el = dims[l - 1], e[l - 1]
            frame += _R(n[l] * pitch(d) * 4)                     # dh_agg
            frame += _R(el * pitch(d) * 4)                       # h_{t-1} per (dst, step)
            if l >= 2:
                frame += _R(el * pitch(d) * 4)                   # dx per (dst, step)
            S3 = lstm_dw_splits(el, d)
            frame += _R(S3 * 4 * d * d * 4) + _R(S3 * pitch(4 * d) * 4)   # dW_ih / dW_hh partials
        if act_dtype == FP32:
            if l >= 2 and not (pool or lstm):
                frame += _R(n[l - 1] * pitch(dims[l]) * 4)      # transposed aggregate of dZ/D
            S = dw_splits(n[l], dims[l], dims[l - 1])
            frame += _R(S * dims[l] * 2 * dims[l - 1] * 4) + _R(S * pitch(dims[l]) * 4)  # dW, db partials
        else:
            if l == L:
                frame += _R(n[l] * pitch(dims[l]) * 2)          # dZ in bf16 (from dlogits)
            if l >= 2:
                frame += 2 * _R(n[l] * pitch(dims[l - 1]) * 2)  # Ys = dZ W_self, Yn = dZ W_neigh / D (bf16)
            S = tc_dw_splits(n[l], dims[l], dims[l - 1])
            Dp = _ceil(dims[l - 1], 64) * 64
            frame += _R(S * dims[l] * 2 * Dp * 4)               # dW partials
            if l == L:
                frame += _R(DB_SPLITS * dims[l] * 4)            # db partials
        bwd = max(bwd, frame)
    lo = blocks + acts + bwd
    hi = blocks + acts + max(bwd, build)
    return lo, hi


# ============================================================================ Eq. 1-2
def grouping_weight(M, I, E, C_ppm):
    """Eq. 1-2: item contribution M_est[i] * R_group[i] with
    R = min(1, I / (O*D*C)), O*D = E (R13), evaluated exactly in integers:
    floor(M * min(1, I*10^6 / (E*C_ppm))).  E = 0 or C_ppm <= 0 => R = 1 (R14)."""
    M, I, E, C_ppm = int(M), int(I), int(E), int(C_ppm)
    if E == 0 or C_ppm <= 0:
        return M
    return min(M, (M * I * 1_000_000) // (E * C_ppm))


def item_stats(g, seeds, L, fanout, seed, dims, act_dtype, aggregator="mean", sharded=False):
    """O, E = sum D, I = unique src of the item's own output block, sizes, M_est (R13, R15)."""
    seeds = np.asarray(seeds, dtype=np.int32)
    n, e = block_sizes(g, seeds, L, fanout, seed)
    lo, hi = mem_model(n, e, dims, act_dtype, aggregator, sharded)
    return dict(O=int(seeds.size), E=int(e[L - 1]), I=int(n[L - 1]), n=n, e=e, M=hi)


def split_explosion(seeds, K):
    """SplitExplosionBucket: K contiguous pieces, numpy.array_split
    sizes (the first O mod K pieces get one extra seed) (R8)."""
    return np.array_split(np.asarray(seeds), K)


def mem_balanced_grouping(items, K, M_ctr):
    """Alg. 4 MemBalancedGrouping (text :343): items sorted by M_est
    descending (ties: bucket degree asc, micro-bucket index asc — R12), each placed into the
    group with the lowest Eq. 2 estimate so far (ties: lowest index); success iff every
    group estimate <= M_ctr.  items: list of dicts with keys d, k, M, w."""
    order = sorted(items, key=lambda it: (-it["M"], it["d"], it["k"]))
    loads = [0] * K
    groups = [[] for _ in range(K)]
    for it in order:
        gi = min(range(K), key=lambda j: (loads[j], j))
        groups[gi].append(it)
        loads[gi] += it["w"]
    return max(loads) <= M_ctr, groups, loads


def _alg3_k_loop(stats, F, piece_stats, mem_budget, C_ppm, k_lo, k_max, fast_paths=True, k_multiple=1):
    """The K loop of Alg. 3 with MemBalancedGrouping (Alg. 4) over the
    per-bucket statistics `stats` {d: dict(M, I, E, O, w, ...)} (non-empty buckets only).
    piece_stats(K) -> [(k, st), ...]: statistics of the K micro-buckets of bucket F (R8).
    For K = k_lo .. k_max: explosion test (R7: K >= 2 and M_est[F] > sum_d M_est[d] / K) ->
    split bucket F into K micro-buckets, else keep it whole; group (Alg. 4); the first K whose
    every group estimate is <= M_ctr wins.
    fast_paths (R25) skips a K without building micro-buckets when sum_{d != F} w_d > K*M_ctr
    and stops at once when a never-split bucket alone exceeds M_ctr; both imply that the plain
    loop (fast_paths=False) fails at that K too, so the result is identical (pinned by
    tests/test_oracle_scheduler.py on random instances).  k_multiple > 1 (reading R31,
    rank-balanced grouping): only multiples of k_multiple are candidates.
    Returns (K, items, groups, loads, exploded) or None."""
    non_split = [d for d in stats if d != F]
    sum_M_all = sum(stats[d]["M"] for d in stats)
    max_w = max([stats[d]["w"] for d in non_split], default=0)
    sum_w = sum(stats[d]["w"] for d in non_split)
    for K in range(k_lo, k_max + 1):
        if k_multiple > 1 and K % k_multiple:
            continue
        if fast_paths:
            if max_w > mem_budget:
                return None                  # a never-split bucket exceeds M_ctr for every K
            if sum_w > K * mem_budget:
                continue                     # some group must exceed M_ctr (weights >= 0)
        items = [dict(d=d, k=0, **stats[d]) for d in non_split]
        exploded = False
        if F in stats:
            exploded = K >= 2 and stats[F]["M"] * K > sum_M_all          # R7
            if exploded:
                for k, st in piece_stats(K):
                    items.append(dict(d=F, k=k, **st))
            else:
                items.append(dict(d=F, k=0, **stats[F]))
        ok, groups, loads = mem_balanced_grouping(items, K, mem_budget)
        if ok:
            return K, items, groups, loads, exploded
    return None


def schedule(g, seeds, L, fanout, F, seed, dims, act_dtype=FP32, mem_budget=INT64_MAX,
             C_ppm=0, k_min=1, k_max=4096, num_gpus=1, aggregator="mean", fast_paths=True, sharded=False,
             k_multiple=1):
    """Alg. 3 Buffalo_Scheduler with the readings of DESIGN.md
    (R7 explosion test, R11 sort/placement keys, R16 K_max, R17 empty groups dropped,
    R24 k_min = #GPUs and LPT rank assignment, R25 fast paths).  Returns a dict plan or None
    (budget)."""
    seeds = np.asarray(seeds, dtype=np.int32)
    f_L = fanout[L - 1]
    D, bucket, order, hist = degree_bucketing(g, seeds, f_L, F)
    pos_of = {d: np.nonzero(bucket == d)[0] for d in range(F + 1)}

    def stats_of(pos):
        st = item_stats(g, seeds[pos], L, fanout, seed, dims, act_dtype, aggregator, sharded)
        st["w"] = grouping_weight(st["M"], st["I"], st["E"], C_ppm)
        st["pos"] = pos
        return st

    stats = {d: stats_of(pos_of[d]) for d in range(F + 1) if pos_of[d].size}

    def piece_stats(K):
        return [(k, stats_of(piece)) for k, piece in enumerate(split_explosion(pos_of[F], K)) if piece.size]

    res = _alg3_k_loop(stats, F, piece_stats, mem_budget, C_ppm, max(k_min, num_gpus, 1), k_max, fast_paths,
                       k_multiple)
    if res is None:
        return None
    K, items, groups, loads, exploded = res
    kept = [(grp, ld) for grp, ld in zip(groups, loads) if grp]
    offsets = [0]
    group_seeds = []
    group_of_seed = np.full(seeds.size, -1, dtype=np.int32)
    for gi, (grp, _) in enumerate(kept):
        for it in sorted(grp, key=lambda it: (it["d"], it["k"])):
            group_seeds.append(seeds[it["pos"]])
            group_of_seed[it["pos"]] = gi
        offsets.append(offsets[-1] + sum(it["O"] for it in grp))
    est = [ld for _, ld in kept]
    rank_load = [0] * max(1, num_gpus)
    rank_of_group = [0] * len(kept)
    for gi in sorted(range(len(kept)), key=lambda j: (-est[j], j)):
        r = min(range(len(rank_load)), key=lambda j: (rank_load[j], j))
        rank_of_group[gi] = r
        rank_load[r] += est[gi]
    return dict(K=len(kept), K_tried=K, exploded=exploded, num_items=len(items),
                group_offsets=np.array(offsets, dtype=np.int64),
                group_seeds=(np.concatenate(group_seeds).astype(np.int32) if group_seeds
                             else np.zeros(0, np.int32)),
                group_of_seed=group_of_seed, est_bytes=np.array(est, dtype=np.int64),
                rank_of_group=np.array(rank_of_group, dtype=np.int32),
                D=D, bucket=bucket, hist=hist)


# ============================================================================ layer math
def mean_adjacency(b):
    """D^-1 A of a block: row i has 1/D(i) at the columns of its sampled neighbours."""
    D = b["D"]
    data = np.repeat(np.where(D > 0, 1.0 / np.maximum(D, 1), 0.0), D)
    return sp.csr_matrix((data, b["col_local"], b["row_ptr"].astype(np.int64)),
                         shape=(b["n_dst"], b["n_src"]))


def round_bf16(x):
    """Round to the nearest bfloat16 (ties to even), returned as float64: keep the top 16 bits
    of the float32 pattern after adding 0x7FFF + lsb (the IEEE round-to-nearest-even rule)."""
    f = np.ascontiguousarray(np.asarray(x, dtype=np.float32))
    u = f.view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).astype(np.float64)


def sage_forward(blocks, X, Ws, bs, storage="fp64"):
    """GraphSAGE-mean forward over the micro-batch's blocks in float64 (Alg. 2 l.8-9):
    h_agg = D^-1 A H_{l-1};  Z_l = [H_{l-1}[:n_l] || h_agg] W_l^T + b_l;  H_l = ReLU(Z_l)
    for l < L, logits = Z_L.  X is the global feature table (indexed via src_global of
    block 1).  storage="bf16" (reading R26) rounds what the bf16 mode stores to bfloat16 — the
    Update operands [H_self || h_agg] and W_l, and H_l — and computes everything else in
    float64, so that the ReLU decisions are taken on the same rounded values as the kernels.
    Returns (logits, cache) with cache for sage_backward."""
    L = len(blocks)
    rnd = round_bf16 if storage == "bf16" else (lambda a: a)
    H = np.asarray(X, dtype=np.float64)[blocks[0]["src_global"]]
    cache = []
    for l in range(1, L + 1):
        b = blocks[l - 1]
        W = rnd(np.asarray(Ws[l - 1], dtype=np.float64))
        d_in = H.shape[1]
        A = mean_adjacency(b)
        agg = rnd(A @ H)
        self_ = rnd(H[: b["n_dst"]])
        Z = self_ @ W[:, :d_in].T + agg @ W[:, d_in:].T + np.asarray(bs[l - 1], dtype=np.float64)
        cache.append(dict(A=A, H_in=H, agg=agg, Z=Z))
        H = rnd(np.maximum(Z, 0.0)) if l < L else Z
    return H, cache


def softmax_ce(logits, y, S):
    """Partial loss of one group, normalised by the global batch size S (R19):
    loss = sum_i CE(softmax(Z_i), y_i) / S; dZ = (softmax - onehot) / S."""
    Z = np.asarray(logits, dtype=np.float64)
    m = Z.max(axis=1, keepdims=True)
    ez = np.exp(Z - m)
    ssum = ez.sum(axis=1, keepdims=True)
    lse = (m + np.log(ssum))[:, 0]
    y = np.asarray(y, dtype=np.int64)
    loss = float(np.sum(lse - Z[np.arange(Z.shape[0]), y]) / S)
    P = ez / ssum
    P[np.arange(Z.shape[0]), y] -= 1.0
    return loss, P / S


def sage_backward(blocks, cache, Ws, dlogits):
    """Backward of sage_forward (Alg. 2 l.11): returns per-layer (dW_l, db_l).
    dZ_L = dlogits; dZ_l = dH_l * 1[Z_l > 0];  dW_l = dZ_l^T [H_{l-1}[:n_l] || h_agg];
    db_l = sum_i dZ_l[i];  dH_{l-1} = pad(dZ_l W_self) + A^T (dZ_l W_neigh)."""
    L = len(blocks)
    grads = [None] * L
    dH = np.asarray(dlogits, dtype=np.float64)
    for l in range(L, 0, -1):
        c = cache[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        d_in = c["H_in"].shape[1]
        dZ = dH if l == L else dH * (c["Z"] > 0)
        n_dst = dZ.shape[0]
        Afwd = np.concatenate([c["H_in"][:n_dst], c["agg"]], axis=1)
        grads[l - 1] = (dZ.T @ Afwd, dZ.sum(axis=0))
        if l > 1:
            dHin = c["A"].T @ (dZ @ W[:, d_in:])
            dHin[:n_dst] += dZ @ W[:, :d_in]
            dH = dHin
    return grads


def pool_forward(blocks, X, Ws, bs, Wps, bps):
    """GraphSAGE-pool forward in float64 (R28; GraphSAGE [16] "pooling aggregator", the
    paper's aggregator list PAPER.md:63).  For block l with input rows H (its src, in local
    order):  Q = H W_pool_l^T + b_pool_l,  P = ReLU(Q);  for dst i and column k,
    h_agg[i,k] = max over the sampled neighbours j of P[j,k] (0 if D(i) = 0), arg[i,k] = the
    neighbour attaining it, the first in CSR order (-1 when the max is 0: no gradient can flow
    there, P = 0 means Q <= 0);  Z = [H[:n_dst] || h_agg] W_l^T + b_l;  H_l = ReLU(Z) for l < L.
    Returns (logits, cache)."""
    L = len(blocks)
    H = np.asarray(X, dtype=np.float64)[blocks[0]["src_global"]]
    cache = []
    for l in range(1, L + 1):
        b = blocks[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        Wp = np.asarray(Wps[l - 1], dtype=np.float64)
        d_in = H.shape[1]
        Q = H @ Wp.T + np.asarray(bps[l - 1], dtype=np.float64)
        P = np.maximum(Q, 0.0)
        n = b["n_dst"]
        agg = np.zeros((n, d_in))
        arg = np.full((n, d_in), -1, dtype=np.int64)
        rp, col = b["row_ptr"], b["col_local"]
        for i in range(n):
            nb = col[rp[i]:rp[i + 1]]
            if len(nb) == 0:
                continue
            vals = P[nb]                                   # [D, d_in]
            first = np.argmax(vals, axis=0)                # first occurrence of the max
            agg[i] = vals[first, np.arange(d_in)]
            arg[i] = np.where(agg[i] > 0, nb[first], -1)
        Z = H[:n] @ W[:, :d_in].T + agg @ W[:, d_in:].T + np.asarray(bs[l - 1], dtype=np.float64)
        cache.append(dict(H_in=H, Q=Q, P=P, agg=agg, arg=arg, Z=Z))
        H = np.maximum(Z, 0.0) if l < L else Z
    return H, cache


def pool_backward(blocks, cache, Ws, Wps, dlogits):
    """Backward of pool_forward: per layer (dW_l, db_l, dW_pool_l, db_pool_l).
    dZ_l = dH_l * 1[Z_l > 0] (dZ_L = dlogits); dW_l = dZ^T [H_self || h_agg]; db_l = sum dZ;
    dh_agg = dZ W_neigh;  dP[j,k] = sum of dh_agg[i,k] over the dst i with arg[i,k] = j;
    dQ = dP * 1[Q > 0];  dW_pool = dQ^T H;  db_pool = sum dQ;
    dH_{l-1} = dQ W_pool + pad(dZ W_self)."""
    L = len(blocks)
    grads = [None] * L
    dH = np.asarray(dlogits, dtype=np.float64)
    for l in range(L, 0, -1):
        c = cache[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        Wp = np.asarray(Wps[l - 1], dtype=np.float64)
        H = c["H_in"]
        d_in = H.shape[1]
        dZ = dH if l == L else dH * (c["Z"] > 0)
        n = dZ.shape[0]
        dW = dZ.T @ np.concatenate([H[:n], c["agg"]], axis=1)
        dagg = dZ @ W[:, d_in:]
        dP = np.zeros_like(c["P"])
        arg = c["arg"]
        for i in range(n):
            for k in range(d_in):
                if arg[i, k] >= 0:
                    dP[arg[i, k], k] += dagg[i, k]
        dQ = dP * (c["Q"] > 0)
        grads[l - 1] = (dW, dZ.sum(axis=0), dQ.T @ H, dQ.sum(axis=0))
        if l > 1:
            dHin = dQ @ Wp
            dHin[:n] += dZ @ W[:, :d_in]
            dH = dHin
    return grads


def _sigmoid(x):
    return 1.0 / (1.0 + np.exp(-x))


def lstm_forward(blocks, X, Ws, bs, Wihs, Whhs, bls):
    """GraphSAGE-LSTM forward in float64 (R29; GraphSAGE [16] LSTM aggregator as DGL's SAGEConv
    'lstm' computes it, PyTorch gate order i, f, g, o).  For block l with input rows H and dst i
    with sampled neighbours j_1..j_D in CSR order: h_0 = c_0 = 0;
    for t = 1..D:  g = W_ih H[j_t] + W_hh h_{t-1} + b;  i = s(g_i), f = s(g_f), u = tanh(g_g),
    o = s(g_o);  c_t = f c_{t-1} + i u;  h_t = o tanh(c_t);   h_agg[i] = h_D (0 if D = 0);
    Z = [H[:n_dst] || h_agg] W_l^T + b_l;  H_l = ReLU(Z) for l < L.
    W_ih, W_hh: [4 d_{l-1}, d_{l-1}], b: [4 d_{l-1}] (= b_ih + b_hh of nn.LSTM)."""
    L = len(blocks)
    H = np.asarray(X, dtype=np.float64)[blocks[0]["src_global"]]
    cache = []
    for l in range(1, L + 1):
        b = blocks[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        Wih = np.asarray(Wihs[l - 1], dtype=np.float64)
        Whh = np.asarray(Whhs[l - 1], dtype=np.float64)
        bl = np.asarray(bls[l - 1], dtype=np.float64)
        d = H.shape[1]
        n = b["n_dst"]
        agg = np.zeros((n, d))
        steps = []                                   # per dst: list of (i, f, u, o, c_prev, c, h_prev)
        rp, col = b["row_ptr"], b["col_local"]
        for r in range(n):
            h = np.zeros(d)
            c = np.zeros(d)
            st = []
            for e in range(rp[r], rp[r + 1]):
                g = Wih @ H[col[e]] + Whh @ h + bl
                gi, gf, gu, go = _sigmoid(g[:d]), _sigmoid(g[d:2 * d]), np.tanh(g[2 * d:3 * d]), _sigmoid(g[3 * d:])
                c_new = gf * c + gi * gu
                h_new = go * np.tanh(c_new)
                st.append((gi, gf, gu, go, c, c_new, h))
                h, c = h_new, c_new
            agg[r] = h
            steps.append(st)
        Z = H[:n] @ W[:, :d].T + agg @ W[:, d:].T + np.asarray(bs[l - 1], dtype=np.float64)
        cache.append(dict(H_in=H, agg=agg, steps=steps, Z=Z))
        H = np.maximum(Z, 0.0) if l < L else Z
    return H, cache


def lstm_backward(blocks, cache, Ws, Wihs, Whhs, dlogits):
    """Backward of lstm_forward (back-propagation through the neighbour sequence): per layer
    (dW_l, db_l, dW_ih_l, dW_hh_l, db_lstm_l).  dZ as for mean; dh_agg = dZ W_neigh; per dst,
    for t = D..1: dc += dh o (1 - tanh^2 c_t); gate pre-activation gradients
    di = dc u i(1-i), df = dc c_{t-1} f(1-f), du = dc i (1-u^2), do = dh tanh(c_t) o(1-o);
    dW_ih += dg x_t^T, dW_hh += dg h_{t-1}^T, db += dg;  dx_t = W_ih^T dg (into dH_{l-1}[j_t]);
    dh <- W_hh^T dg, dc <- dc f.   dH_{l-1} = (sum of dx over edges) + pad(dZ W_self)."""
    L = len(blocks)
    grads = [None] * L
    dH = np.asarray(dlogits, dtype=np.float64)
    for l in range(L, 0, -1):
        c_ = cache[l - 1]
        b = blocks[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        Wih = np.asarray(Wihs[l - 1], dtype=np.float64)
        Whh = np.asarray(Whhs[l - 1], dtype=np.float64)
        H = c_["H_in"]
        d = H.shape[1]
        dZ = dH if l == L else dH * (c_["Z"] > 0)
        n = dZ.shape[0]
        dW = dZ.T @ np.concatenate([H[:n], c_["agg"]], axis=1)
        dagg = dZ @ W[:, d:]
        dWih = np.zeros_like(Wih)
        dWhh = np.zeros_like(Whh)
        dbl = np.zeros(4 * d)
        dHin = np.zeros_like(H)
        rp, col = b["row_ptr"], b["col_local"]
        for r in range(n):
            dh = dagg[r].copy()
            dc = np.zeros(d)
            st = c_["steps"][r]
            for t in range(len(st) - 1, -1, -1):
                gi, gf, gu, go, c_prev, c_t, h_prev = st[t]
                tc = np.tanh(c_t)
                dc = dc + dh * go * (1.0 - tc * tc)
                dg = np.concatenate([dc * gu * gi * (1.0 - gi), dc * c_prev * gf * (1.0 - gf),
                                     dc * gi * (1.0 - gu * gu), dh * tc * go * (1.0 - go)])
                x = H[col[rp[r] + t]]
                dWih += np.outer(dg, x)
                dWhh += np.outer(dg, h_prev)
                dbl += dg
                dHin[col[rp[r] + t]] += Wih.T @ dg
                dh = Whh.T @ dg
                dc = dc * gf
        grads[l - 1] = (dW, dZ.sum(axis=0), dWih, dWhh, dbl)
        if l > 1:
            dHin[:n] += dZ @ W[:, :d]
            dH = dHin
    return grads


def gat_forward(blocks, X, Ws, bs, als, ars, slope=0.2):
    """GAT forward in float64 (R30; one head per layer, as DGL's GATConv computes it with
    allow_zero_in_degree).  For block l with input rows H (its src): Z = H W_l^T;
    el[j] = a_l . Z[j] (every src), er[i] = a_r . Z[i] (dst, the prefix of src);
    s_ij = LeakyReLU(el[j] + er[i]);  alpha_ij = softmax of s_ij over the sampled neighbours j
    of i;  out_i = sum_j alpha_ij Z[j] + b_l (b_l alone when D(i) = 0);  H_l = ELU(out) for
    l < L, logits = out at l = L.  W_l: [d_l, d_{l-1}], a_l, a_r, b_l: [d_l]."""
    L = len(blocks)
    H = np.asarray(X, dtype=np.float64)[blocks[0]["src_global"]]
    cache = []
    for l in range(1, L + 1):
        b = blocks[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        al = np.asarray(als[l - 1], dtype=np.float64)
        ar = np.asarray(ars[l - 1], dtype=np.float64)
        Z = H @ W.T
        el = Z @ al
        n = b["n_dst"]
        er = Z[:n] @ ar
        rp, col = b["row_ptr"], b["col_local"]
        alpha = np.zeros(b["n_edges"])
        out = np.tile(np.asarray(bs[l - 1], dtype=np.float64), (n, 1))
        for i in range(n):
            e0, e1 = rp[i], rp[i + 1]
            if e1 == e0:
                continue
            sc = el[col[e0:e1]] + er[i]
            sc = np.where(sc > 0, sc, slope * sc)
            w = np.exp(sc - sc.max())
            alpha[e0:e1] = w / w.sum()
            out[i] += alpha[e0:e1] @ Z[col[e0:e1]]
        cache.append(dict(H_in=H, Z=Z, el=el, er=er, alpha=alpha, out=out))
        H = np.where(out > 0, out, np.expm1(out)) if l < L else out
    return H, cache


def gat_backward(blocks, cache, Ws, als, ars, dlogits, slope=0.2):
    """Backward of gat_forward: per layer (dW_l, db_l, da_l, da_r).
    dOut = dH * ELU'(out) (dOut_L = dlogits);  db = sum dOut;  dZ[j] = sum_i alpha_ij dOut_i;
    dalpha_ij = dOut_i . Z[j];  ds_ij = alpha_ij (dalpha_ij - sum_k alpha_ik dalpha_ik) * LeakyReLU';
    dZ[j] += (sum_i ds_ij) a_l;  dZ[i] += (sum_j ds_ij) a_r;  da_l = sum_j (sum_i ds_ij) Z[j];
    da_r = sum_i (sum_j ds_ij) Z[i];  dW = dZ^T H;  dH_{l-1} = dZ W."""
    L = len(blocks)
    grads = [None] * L
    dH = np.asarray(dlogits, dtype=np.float64)
    for l in range(L, 0, -1):
        c = cache[l - 1]
        b = blocks[l - 1]
        W = np.asarray(Ws[l - 1], dtype=np.float64)
        al = np.asarray(als[l - 1], dtype=np.float64)
        ar = np.asarray(ars[l - 1], dtype=np.float64)
        out, Z, alpha = c["out"], c["Z"], c["alpha"]
        dO = dH if l == L else dH * np.where(out > 0, 1.0, np.exp(out))
        n = dO.shape[0]
        rp, col = b["row_ptr"], b["col_local"]
        dZ = np.zeros_like(Z)
        d_el = np.zeros(Z.shape[0])
        d_er = np.zeros(n)
        for i in range(n):
            e0, e1 = rp[i], rp[i + 1]
            if e1 == e0:
                continue
            nb = col[e0:e1]
            a = alpha[e0:e1]
            dZ[nb] += np.outer(a, dO[i])
            da = Z[nb] @ dO[i]
            de = a * (da - a @ da)
            sc = c["el"][nb] + c["er"][i]
            ds = de * np.where(sc > 0, 1.0, slope)
            d_er[i] = ds.sum()
            np.add.at(d_el, nb, ds)
        dZ += np.outer(d_el, al)
        dZ[:n] += np.outer(d_er, ar)
        grads[l - 1] = (dZ.T @ c["H_in"], dO.sum(axis=0), d_el @ Z, d_er @ Z[:n])
        if l > 1:
            dH = dZ @ W
    return grads


def microbatch_step(g, seeds_k, X, y, Ws, bs, L, fanout, seed, S, storage="fp64"):
    """One micro-batch of Alg. 2 (l.4-12): blocks, forward, partial loss, gradients."""
    blocks = build_blocks(g, seeds_k, L, fanout, seed)
    logits, cache = sage_forward(blocks, X, Ws, bs, storage)
    loss, dlog = softmax_ce(logits, y[np.asarray(seeds_k)], S)
    grads = sage_backward(blocks, cache, Ws, dlog)
    return loss, grads, blocks


def train_epoch(g, seeds, X, y, Ws, bs, L, fanout, F, seed, dims, lr=0.0, storage="fp64", **sched_kw):
    """Alg. 2: schedule, then every group's forward/backward with the
    partial gradients accumulated, then ONE optimizer step (SGD with rate lr, R18)."""
    plan = schedule(g, seeds, L, fanout, F, seed, dims, **sched_kw)
    if plan is None:
        raise RuntimeError("Buffalo scheduler: no K satisfies the memory budget")
    S = len(seeds)
    total = 0.0
    acc = [(np.zeros_like(np.asarray(W, np.float64)), np.zeros(len(b))) for W, b in zip(Ws, bs)]
    off = plan["group_offsets"]
    for k in range(plan["K"]):
        sk = plan["group_seeds"][off[k]:off[k + 1]]
        loss, grads, _ = microbatch_step(g, sk, X, y, Ws, bs, L, fanout, seed, S, storage)
        total += loss
        acc = [(a + gw, b + gb) for (a, b), (gw, gb) in zip(acc, grads)]
    newW = [np.asarray(W, np.float64) - lr * gW for W, (gW, _) in zip(Ws, acc)]
    newb = [np.asarray(b, np.float64) - lr * gb for b, (_, gb) in zip(bs, acc)]
    return total, acc, newW, newb, plan


# ============================================================================ clustering (Eq. 1's C)
def triangles(g, nodes=None):
    """T_v = number of adjacent pairs among the neighbours of v (triangles through v), by
    definition (oracle_triangles, every neighbour pair tested).  nodes=None: all nodes."""
    if nodes is None:
        T = np.zeros(g.N, dtype=np.int64)
        lib().oracle_triangles(_p(g.row_ptr), _p(g.col), 0, g.N, _p(T))
        return T
    out = np.zeros(len(nodes), dtype=np.int64)
    one = np.zeros(1, dtype=np.int64)
    for i, v in enumerate(nodes):
        lib().oracle_triangles(_p(g.row_ptr), _p(g.col), int(v), int(v) + 1, _p(one))
        out[i] = one[0]
    return out


def avg_clustering(g, T=None):
    """Average clustering coefficient C (reading R27): the mean over ALL nodes of the local
    coefficient 2 T_v / (d_v (d_v - 1)), taken as 0 for d_v < 2 (Newman [27]; networkx's
    average_clustering with count_zeros=True).  float64, summed in node order."""
    T = triangles(g) if T is None else np.asarray(T, np.int64)
    d = np.diff(np.asarray(g.row_ptr, np.int64)).astype(np.float64)
    loc = np.zeros(g.N, dtype=np.float64)
    ok = d >= 2
    loc[ok] = 2.0 * T[ok] / (d[ok] * (d[ok] - 1.0))
    total = 0.0
    for x in loc:                      # plain sequential sum (node order)
        total += x
    return total / g.N
