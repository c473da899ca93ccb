"""Thin ctypes binding of include/buffalo.h (argument marshalling only).

Every function here forwards to libbuffalo.so with the same name minus the `buffalo_` prefix.
Device buffers are torch CUDA tensors (PyTorch is used for device memory and streams only);
there is no CPU fallback: loading fails loudly without the built library or a GPU.
"""
import ctypes
import os

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# BUFFALO_LIB: load an experimental build instead (diagnostics only; tools/exp_build.sh)
LIB_PATH = os.environ.get("BUFFALO_LIB") or os.path.join(_HERE, "libbuffalo.so")

c_i32, c_i64, c_u64, c_p, c_sz, c_f = (ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64,
                                       ctypes.c_void_p, ctypes.c_size_t, ctypes.c_float)

OK, ERR_INVALID_ARG, ERR_BUDGET, ERR_CAPACITY, ERR_CUDA, ERR_UNSUPPORTED = range(6)
FP32, BF16 = 0, 1
GEMM_FFMA, GEMM_BF16 = 0, 1
AGG_MEAN, AGG_POOL, AGG_LSTM, AGG_GAT = 0, 1, 2, 3
MAX_LAYERS = 8

EXPORTS = [
    "buffalo_graph_workspace_bytes", "buffalo_graph_prepare", "buffalo_bucketize_workspace_bytes",
    "buffalo_bucketize", "buffalo_build_blocks", "buffalo_packed_weight_bytes",
    "buffalo_pack_weights", "buffalo_sage_fwd", "buffalo_softmax_ce",
    "buffalo_sage_bwd_scratch_bytes", "buffalo_sage_bwd", "buffalo_sgd_step",
    "buffalo_estimate_mem", "buffalo_launch_count", "buffalo_profile_begin", "buffalo_profile_end",
    "buffalo_status_str", "buffalo_last_error",
    "buffalo_clustering_workspace_bytes", "buffalo_triangles", "buffalo_avg_clustering",
    "buffalo_pool_fwd", "buffalo_pool_bwd", "buffalo_lstm_fwd", "buffalo_lstm_bwd",
    "buffalo_gat_fwd", "buffalo_gat_bwd", "buffalo_graph_validate",
    "buffalo_ipc_export", "buffalo_ipc_open", "buffalo_ipc_close",
]


class BuffaloError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_STATUS = {0: "BUFFALO_OK", 1: "BUFFALO_ERR_INVALID_ARG", 2: "BUFFALO_ERR_BUDGET",
           3: "BUFFALO_ERR_CAPACITY", 4: "BUFFALO_ERR_CUDA", 5: "BUFFALO_ERR_UNSUPPORTED"}


class Graph(ctypes.Structure):
    _fields_ = [("num_nodes", c_i64), ("nnz", c_i64), ("row_ptr", c_p), ("col", c_p), ("node_map", c_p)]


class Sampler(ctypes.Structure):
    _fields_ = [("num_layers", c_i32), ("fanout", c_i32 * MAX_LAYERS), ("cutoff_F", c_i32), ("seed", c_u64),
                ("cache", c_p * MAX_LAYERS)]


MAX_SHARDS = 8
IPC_HANDLE_BYTES = 72


class FeatureShards(ctypes.Structure):
    _fields_ = [("num_shards", c_i32), ("rows_per_shard", c_i64), ("shard", c_p * MAX_SHARDS)]


class Model(ctypes.Structure):
    _fields_ = [("num_layers", c_i32), ("dim", c_i32 * (MAX_LAYERS + 1)), ("feat_dtype", c_i32),
                ("gemm_mode", c_i32), ("feat_pitch", c_i64), ("aggregator", c_i32),
                ("feat_shards", ctypes.POINTER(FeatureShards))]


ALLGATHER_FN = ctypes.CFUNCTYPE(c_i32, c_p, c_p, c_p, c_i64)


class Sched(ctypes.Structure):
    _fields_ = [("mem_budget", c_i64), ("C_ppm", c_i64), ("k_min", c_i32), ("k_max", c_i32),
                ("num_gpus", c_i32), ("k_multiple", c_i32), ("rank", c_i32), ("allgather", ALLGATHER_FN),
                ("allgather_ctx", c_p)]


class Plan(ctypes.Structure):
    _fields_ = [("group_of_seed", c_p), ("group_seeds", c_p), ("group_offsets", c_p),
                ("group_offsets_h", c_p), ("est_bytes_h", c_p), ("rank_of_group_h", c_p),
                ("hist_h", c_p), ("group_sizes_h", c_p), ("k_out", c_i32), ("k_tried", c_i32), ("exploded", c_i32),
                ("num_items", c_i32)]


class Block(ctypes.Structure):
    _fields_ = [("n_dst", c_i64), ("n_src", c_i64), ("n_edges", c_i64), ("n_heavy", c_i64),
                ("n_heavy_t", c_i64),
                ("row_ptr", c_p), ("col_local", c_p), ("col_global", c_p), ("src_global", c_p),
                ("t_row_ptr", c_p), ("t_col", c_p), ("heavy", c_p), ("cls_perm", c_p), ("t_perm", c_p),
                ("agg", c_p), ("out", c_p), ("dh", c_p), ("bwd_scratch", c_p),
                ("ld_agg", c_i64), ("ld_out", c_i64), ("ld_dh", c_i64), ("bwd_scratch_bytes", c_i64),
                ("pool_P", c_p), ("pool_arg", c_p), ("ld_pool", c_i64),
                ("agg_saved", c_p), ("agg_saved_bytes", c_i64), ("fanout", c_i64),
                ("self_rows", c_p), ("ld_self", c_i64)]


class Blocks(ctypes.Structure):
    _fields_ = [("num_layers", c_i32), ("layer", Block * MAX_LAYERS), ("arena_used", c_i64),
                ("arena_peak", c_i64), ("est_lo", c_i64), ("est_hi", c_i64)]


_lib = None


def lib(require_gpu=True):
    """Load libbuffalo.so (raises if it is missing or, with require_gpu, if there is no GPU)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libbuffalo.so not built ({LIB_PATH}); run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        P = c_p
        sig = {
            "buffalo_graph_workspace_bytes": (c_sz, [c_i64]),
            "buffalo_graph_prepare": (c_i32, [P, P, c_sz, P]),
            "buffalo_bucketize_workspace_bytes": (c_sz, [P, c_i64, P, P]),
            "buffalo_bucketize": (c_i32, [P, P, c_i64, P, P, P, P, P, c_sz, P]),
            "buffalo_build_blocks": (c_i32, [P, P, c_i64, P, P, P, P, c_sz, P, P, P]),
            "buffalo_packed_weight_bytes": (c_sz, [P, c_i32]),
            "buffalo_pack_weights": (c_i32, [P, c_i32, P, P, P]),
            "buffalo_sage_fwd": (c_i32, [P, c_i32, P, P, c_i64, P, P, P, P, c_i64, P, c_i64, P]),
            "buffalo_softmax_ce": (c_i32, [P, c_i64, c_i64, c_i32, P, P, c_i64, P, P, c_i64, P]),
            "buffalo_sage_bwd_scratch_bytes": (c_sz, [P, c_i32, P]),
            "buffalo_sage_bwd": (c_i32, [P, c_i32, P, P, c_i64, P, c_i64, P, c_i64, P, c_i64, P, P,
                                         P, P, P, c_i64, P, c_sz, P]),
            "buffalo_sgd_step": (c_i32, [P, P, c_i64, c_f, P]),
            "buffalo_estimate_mem": (c_i32, [c_i32, P, P, P, P, P]),
            "buffalo_launch_count": (c_i64, []),
            "buffalo_profile_begin": (c_i32, [ctypes.c_char_p, P, c_i64, P]),
            "buffalo_profile_end": (c_i32, [P, P, P]),
            "buffalo_clustering_workspace_bytes": (c_sz, [P]),
            "buffalo_triangles": (c_i32, [P, P, P, c_sz, P]),
            "buffalo_avg_clustering": (c_i32, [P, P, P, P, P, c_sz, P]),
            "buffalo_pool_fwd": (c_i32, [P, c_i32, P, P, c_i64, P, P, P, P, P, P, c_i64, P, c_i64, P, P, c_i64, P]),
            "buffalo_pool_bwd": (c_i32, [P, c_i32, P, P, c_i64, P, c_i64, P, c_i64, P, c_i64, P, P, c_i64, P, P,
                                         P, P, P, P, P, c_i64, P, c_sz, P]),
            "buffalo_lstm_fwd": (c_i32, [P, c_i32, P, P, c_i64, P, P, P, P, P, P, P, c_i64, P, c_i64, P, c_sz, P]),
            "buffalo_lstm_bwd": (c_i32, [P, c_i32, P, P, c_i64, P, c_i64, P, c_i64, P, c_i64, P, c_sz, P, P, P,
                                         P, P, P, P, P, P, c_i64, P, c_sz, P]),
            "buffalo_gat_fwd": (c_i32, [P, c_i32, P, P, c_i64, P, P, P, P, P, c_i64, P, c_sz, P]),
            "buffalo_gat_bwd": (c_i32, [P, c_i32, P, P, c_i64, P, c_i64, P, c_i64, P, c_sz, P, P, P, P, P, P, P, P,
                                        c_i64, P, c_sz, P]),
            "buffalo_graph_validate": (c_i32, [P, c_i32, P]),
            "buffalo_ipc_export": (c_i32, [P, P]),
            "buffalo_ipc_open": (c_i32, [P, P]),
            "buffalo_ipc_close": (c_i32, [P, P]),
            "buffalo_status_str": (ctypes.c_char_p, [c_i32]),
            "buffalo_last_error": (ctypes.c_char_p, []),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    if require_gpu and not torch.cuda.is_available():
        raise RuntimeError("libbuffalo needs a CUDA device (sm_100a); there is no CPU fallback")
    return _lib


def _check(status):
    if status != OK:
        raise BuffaloError(status, lib(False).buffalo_last_error().decode())


def ptr(t):
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def dev(t, dtypes, name):
    """Pointer of a device tensor argument after checking what the C ABI assumes of it: a CUDA,
    C-contiguous tensor of one of `dtypes` (an int64 tensor read as int32 ids, or an fp32 table
    read as bf16, would otherwise give wrong results silently).  Raw ints pass through."""
    if t is None or isinstance(t, int):
        return t
    if not (t.is_cuda and t.is_contiguous()):
        raise ValueError(f"{name}: expected a contiguous CUDA tensor")
    if t.dtype not in dtypes:
        raise TypeError(f"{name}: dtype {t.dtype}, expected {' or '.join(str(d) for d in dtypes)}")
    return t.data_ptr()


I32 = (torch.int32,)
F32 = (torch.float32,)
FEAT = {FP32: (torch.float32,), BF16: (torch.bfloat16,)}


def act_dtypes(model, layer):
    """dtype of layer `layer`'s input rows: the feature table at layer 1, else the activations."""
    if layer == 1:
        return FEAT[model.feat_dtype]
    return (torch.bfloat16,) if model.gemm_mode == GEMM_BF16 else (torch.float32,)


def stream_ptr(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


def ref(x):
    return ctypes.byref(x) if x is not None else None


# ------------------------------------------------------------------------- wrappers
def graph_workspace_bytes(num_nodes):
    return lib(False).buffalo_graph_workspace_bytes(num_nodes)


def graph_prepare(graph, workspace, stream=None):
    _check(lib().buffalo_graph_prepare(ref(graph), ptr(workspace), workspace.numel() * workspace.element_size(),
                                       stream_ptr(stream)))


def graph_validate(graph, check_symmetric=True, stream=None):
    """O(N + nnz) check of the CSR contract on the device (raises BuffaloError)."""
    _check(lib().buffalo_graph_validate(ref(graph), int(bool(check_symmetric)), stream_ptr(stream)))


def bucketize_workspace_bytes(graph, n_seeds, sampler, model):
    return lib(False).buffalo_bucketize_workspace_bytes(ref(graph), n_seeds, ref(sampler), ref(model))


def bucketize(graph, seeds, sampler, model, sched, plan, workspace, stream=None):
    _check(lib().buffalo_bucketize(ref(graph), dev(seeds, I32, "seeds"), seeds.numel(), ref(sampler), ref(model),
                                   ref(sched), ref(plan), ptr(workspace), workspace.numel(),
                                   stream_ptr(stream)))


def build_blocks(graph, group_seeds, n, sampler, model, blocks, arena, sizes=None, stream=None):
    """Returns BUFFALO_OK or raises; on BUFFALO_ERR_CAPACITY the error carries .required.
    sizes: None or a C-contiguous int64 numpy row [2L+1] of plan.group_sizes_h (sync-free build)."""
    req = c_i64(0)
    sz = None
    if sizes is not None:
        assert sizes.dtype == np.int64 and sizes.flags["C_CONTIGUOUS"]
        sz = sizes.ctypes.data
    st = lib().buffalo_build_blocks(ref(graph), dev(group_seeds, I32, "group_seeds"), n, ref(sampler), ref(model),
                                    ref(blocks), ptr(arena), arena.numel(), ctypes.byref(req), sz,
                                    stream_ptr(stream))
    if st == ERR_CAPACITY:
        err = BuffaloError(st, lib(False).buffalo_last_error().decode())
        err.required = req.value
        raise err
    _check(st)
    return req.value


def packed_weight_bytes(model, layer):
    return lib(False).buffalo_packed_weight_bytes(ref(model), layer)


def pack_weights(model, layer, W, packed, stream=None):
    _check(lib().buffalo_pack_weights(ref(model), layer, ptr(W), ptr(packed), stream_ptr(stream)))


def sage_fwd(blk, layer, model, h_src, ld_src, W, W_packed, b, out, ld_out, saved_agg, ld_agg, stream=None):
    _check(lib().buffalo_sage_fwd(ref(blk), layer, ref(model), dev(h_src, act_dtypes(model, layer), "h_src"), ld_src,
                                  dev(W, F32, "W"), ptr(W_packed),
                                  ptr(b), ptr(out), ld_out, ptr(saved_agg), ld_agg, stream_ptr(stream)))


def softmax_ce(logits, ld, n, classes, labels, row_ids, batch_size, loss_accum, dlogits, ld_d, stream=None):
    _check(lib().buffalo_softmax_ce(ptr(logits), ld, n, classes, dev(labels, I32, "labels"),
                                    dev(row_ids, I32, "row_ids"), batch_size,
                                    ptr(loss_accum), ptr(dlogits), ld_d, stream_ptr(stream)))


def sage_bwd_scratch_bytes(blk, layer, model):
    return lib(False).buffalo_sage_bwd_scratch_bytes(ref(blk), layer, ref(model))


def sage_bwd(blk, layer, model, dh_dst, ld_dh, h_src, ld_src, saved_agg, ld_agg, h_dst, ld_hdst, W,
             W_packed, dW, db, dh_src, ld_dh_src, scratch, scratch_bytes, stream=None):
    _check(lib().buffalo_sage_bwd(ref(blk), layer, ref(model), ptr(dh_dst), ld_dh,
                                  dev(h_src, act_dtypes(model, layer), "h_src"), ld_src,
                                  ptr(saved_agg), ld_agg, ptr(h_dst), ld_hdst, ptr(W), ptr(W_packed),
                                  ptr(dW), ptr(db), ptr(dh_src), ld_dh_src, ptr(scratch),
                                  scratch_bytes, stream_ptr(stream)))


def pool_fwd(blk, layer, model, h_src, ld_src, W_pool, b_pool, W, W_packed, b, out, ld_out, saved_agg, ld_agg,
             P, arg, ld_pool, stream=None):
    _check(lib().buffalo_pool_fwd(ref(blk), layer, ref(model), dev(h_src, act_dtypes(model, layer), "h_src"), ld_src, ptr(W_pool), ptr(b_pool), ptr(W),
                                  ptr(W_packed), ptr(b), ptr(out), ld_out, ptr(saved_agg), ld_agg, ptr(P), ptr(arg),
                                  ld_pool, stream_ptr(stream)))


def pool_bwd(blk, layer, model, dh_dst, ld_dh, h_src, ld_src, saved_agg, ld_agg, h_dst, ld_hdst, P, arg, ld_pool,
             W_pool, W, dW_pool, db_pool, dW, db, dh_src, ld_dh_src, scratch, scratch_bytes, stream=None):
    _check(lib().buffalo_pool_bwd(ref(blk), layer, ref(model), ptr(dh_dst), ld_dh,
                                  dev(h_src, act_dtypes(model, layer), "h_src"), ld_src,
                                  ptr(saved_agg), ld_agg, ptr(h_dst), ld_hdst, ptr(P), ptr(arg), ld_pool,
                                  ptr(W_pool), ptr(W), ptr(dW_pool), ptr(db_pool), ptr(dW), ptr(db), ptr(dh_src),
                                  ld_dh_src, ptr(scratch), scratch_bytes, stream_ptr(stream)))


def lstm_fwd(blk, layer, model, h_src, ld_src, W_ih, W_hh, b_lstm, W, W_packed, b, out, ld_out, saved_agg, ld_agg,
             stream=None):
    _check(lib().buffalo_lstm_fwd(ref(blk), layer, ref(model), dev(h_src, act_dtypes(model, layer), "h_src"), ld_src, ptr(W_ih), ptr(W_hh), ptr(b_lstm),
                                  ptr(W), ptr(W_packed), ptr(b), ptr(out), ld_out, ptr(saved_agg), ld_agg,
                                  ptr(blk.agg_saved), blk.agg_saved_bytes, stream_ptr(stream)))


def lstm_bwd(blk, layer, model, dh_dst, ld_dh, h_src, ld_src, saved_agg, ld_agg, h_dst, ld_hdst, W_ih, W_hh, W,
             dW_ih, dW_hh, db_lstm, dW, db, dh_src, ld_dh_src, scratch, scratch_bytes, stream=None):
    _check(lib().buffalo_lstm_bwd(ref(blk), layer, ref(model), ptr(dh_dst), ld_dh,
                                  dev(h_src, act_dtypes(model, layer), "h_src"), ld_src,
                                  ptr(saved_agg), ld_agg, ptr(h_dst), ld_hdst, ptr(blk.agg_saved),
                                  blk.agg_saved_bytes, ptr(W_ih), ptr(W_hh), ptr(W), ptr(dW_ih), ptr(dW_hh),
                                  ptr(db_lstm), ptr(dW), ptr(db), ptr(dh_src), ld_dh_src, ptr(scratch),
                                  scratch_bytes, stream_ptr(stream)))


def gat_fwd(blk, layer, model, h_src, ld_src, W, a_l, a_r, b, out, ld_out, stream=None):
    _check(lib().buffalo_gat_fwd(ref(blk), layer, ref(model), dev(h_src, act_dtypes(model, layer), "h_src"), ld_src, ptr(W), ptr(a_l), ptr(a_r), ptr(b),
                                 ptr(out), ld_out, ptr(blk.agg_saved), blk.agg_saved_bytes, stream_ptr(stream)))


def gat_bwd(blk, layer, model, dh_dst, ld_dh, h_src, ld_src, h_dst, ld_hdst, W, a_l, a_r, dW, db, da_l, da_r,
            dh_src, ld_dh_src, scratch, scratch_bytes, stream=None):
    _check(lib().buffalo_gat_bwd(ref(blk), layer, ref(model), ptr(dh_dst), ld_dh,
                                  dev(h_src, act_dtypes(model, layer), "h_src"), ld_src, ptr(h_dst),
                                 ld_hdst, ptr(blk.agg_saved), blk.agg_saved_bytes, ptr(W), ptr(a_l), ptr(a_r),
                                 ptr(dW), ptr(db), ptr(da_l), ptr(da_r), ptr(dh_src), ld_dh_src, ptr(scratch),
                                 scratch_bytes, stream_ptr(stream)))


def sgd_step(param, grad, lr, stream=None):
    _check(lib().buffalo_sgd_step(ptr(param), ptr(grad), param.numel(), lr, stream_ptr(stream)))


def estimate_mem(n, e, model):
    L = len(e)
    na = (c_i64 * (L + 1))(*n)
    ea = (c_i64 * L)(*e)
    lo, hi = c_i64(0), c_i64(0)
    _check(lib(False).buffalo_estimate_mem(L, na, ea, ref(model), ctypes.byref(lo), ctypes.byref(hi)))
    return lo.value, hi.value


def clustering_workspace_bytes(graph):
    return lib(False).buffalo_clustering_workspace_bytes(ref(graph))


def triangles(graph, T, workspace, stream=None):
    """T (int64 CUDA tensor [N]) = triangles through each node (C of Eq. 1, R27)."""
    _check(lib().buffalo_triangles(ref(graph), ptr(T), ptr(workspace), workspace.numel() * workspace.element_size(),
                                   stream_ptr(stream)))


def avg_clustering(graph, T, workspace, stream=None):
    """(C, C_ppm) from T (synchronises once)."""
    C, ppm = ctypes.c_double(0), c_i64(0)
    _check(lib().buffalo_avg_clustering(ref(graph), ptr(T), ctypes.byref(C), ctypes.byref(ppm), ptr(workspace),
                                        workspace.numel() * workspace.element_size(), stream_ptr(stream)))
    return C.value, ppm.value


def clustering(graph, stream=None):
    """Triangles per node and C for a buffalo Graph struct: (T tensor, C, C_ppm).  Allocates the
    workspace and T with torch (device memory only)."""
    ws = torch.empty(clustering_workspace_bytes(graph), dtype=torch.uint8, device="cuda")
    T = torch.empty(graph.num_nodes, dtype=torch.int64, device="cuda")
    triangles(graph, T, ws, stream)
    C, ppm = avg_clustering(graph, T, ws, stream)
    return T, C, ppm


def ipc_export(t):
    """IPC handle (bytes) of the device memory at tensor t's data pointer."""
    buf = ctypes.create_string_buffer(IPC_HANDLE_BYTES)
    _check(lib().buffalo_ipc_export(ptr(t), buf))
    return buf.raw


def ipc_open(handle):
    """Device pointer (int) of a peer's memory from its handle (lazy NVLink peer access)."""
    out = c_p(0)
    _check(lib().buffalo_ipc_open(ctypes.create_string_buffer(bytes(handle), IPC_HANDLE_BYTES), ctypes.byref(out)))
    return out.value


def ipc_close(handle, p):
    _check(lib().buffalo_ipc_close(ctypes.create_string_buffer(bytes(handle), IPC_HANDLE_BYTES), p))


def launch_count():
    return lib(False).buffalo_launch_count()


def profile_begin(family, counters, stream=None):
    """Times every launch of a kernel family (diagnostic; counters: int64 CUDA tensor)."""
    _check(lib().buffalo_profile_begin(family.encode(), ptr(counters), counters.numel(), stream_ptr(stream)))


def profile_end():
    """(summed launch ms, number of launches, algorithmic bytes) of the profiled family."""
    ms, n, by = ctypes.c_double(0), c_i64(0), ctypes.c_double(0)
    _check(lib().buffalo_profile_end(ctypes.byref(ms), ctypes.byref(n), ctypes.byref(by)))
    return ms.value, n.value, by.value


# ------------------------------------------------------------------------- struct helpers
def make_sampler(fanout, F, seed, cache=None):
    """cache: None or a list of per-block int32 CUDA tensors [num_nodes * fanout] (None entries
    allowed), the optional sample cache of include/buffalo.h."""
    s = Sampler()
    for i, c in enumerate(cache or []):
        s.cache[i] = ptr(c) if c is not None else None
    s.num_layers = len(fanout)
    for i, f in enumerate(fanout):
        s.fanout[i] = int(f)
    s.cutoff_F = int(F)
    s.seed = int(seed)
    return s


def make_shards(pointers, rows_per_shard):
    """buffalo_feature_shards for a node-id-range sharded table (device pointers / tensors)."""
    s = FeatureShards()
    if not 1 <= len(pointers) <= MAX_SHARDS:
        raise ValueError(f"1..{MAX_SHARDS} shards")
    s.num_shards = len(pointers)
    s.rows_per_shard = int(rows_per_shard)
    for i, p in enumerate(pointers):
        s.shard[i] = ptr(p)
    return s


def make_model(dims, feat_dtype=FP32, gemm_mode=GEMM_FFMA, feat_pitch=None, aggregator=AGG_MEAN, shards=None):
    """shards: None or a FeatureShards struct (kept alive by the returned model)."""
    m = Model()
    if shards is not None:
        m.feat_shards = ctypes.pointer(shards)
        m._shards_ref = shards
    m.num_layers = len(dims) - 1
    for i, d in enumerate(dims):
        m.dim[i] = int(d)
    m.feat_dtype = feat_dtype
    m.gemm_mode = gemm_mode
    m.feat_pitch = int(feat_pitch if feat_pitch else ((dims[0] + 7) // 8) * 8)
    m.aggregator = int(aggregator)
    return m


def make_sched(mem_budget=(1 << 63) - 1, C_ppm=0, k_min=1, k_max=4096, num_gpus=1, k_multiple=1, rank=0,
               allgather=None):
    """allgather: None or an ALLGATHER_FN (kept alive by the returned struct)."""
    s = Sched()
    s.mem_budget, s.C_ppm, s.k_min, s.k_max, s.num_gpus = int(mem_budget), int(C_ppm), k_min, k_max, num_gpus
    s.k_multiple = int(k_multiple)
    s.rank = int(rank)
    if allgather is not None:
        s.allgather = allgather
        s._allgather_ref = allgather
    return s


def make_allgather(world, group=None, device=None):
    """An ALLGATHER_FN over torch.distributed (host buffers; NCCL groups go through `device`)."""
    import torch.distributed as dist

    def fn(ctx, send, recv, nbytes):
        try:
            src = torch.frombuffer((ctypes.c_char * nbytes).from_address(send), dtype=torch.uint8).clone()
            if device is not None:
                src = src.to(device)
            out = torch.empty(world * nbytes, dtype=torch.uint8, device=src.device)
            dist.all_gather_into_tensor(out, src, group=group)
            out = out.cpu().contiguous()
            ctypes.memmove(recv, out.data_ptr(), world * nbytes)
            return 0
        except Exception:                    # noqa: BLE001 (reported to the library as a failure)
            return 1
    return ALLGATHER_FN(fn)


def pitch(d):
    return ((int(d) + 7) // 8) * 8
