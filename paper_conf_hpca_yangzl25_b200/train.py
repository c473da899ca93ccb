"""Epoch driver: one Buffalo iteration (Alg. 2) through the C ABI.

Python only allocates torch device buffers, marshals arguments and calls NCCL through
torch.distributed for the single gradient allreduce (R24); every step of the
path (bucketize, blocks, forward, loss, backward, optimizer) runs in libbuffalo's kernels.
"""
import ctypes
import time

import numpy as np
import torch

from . import buffalo as B


def own_groups(rank_of_group, rank):
    """Groups this rank runs: those the scheduler's LPT assignment gave it (R24)."""
    return [k for k in range(len(rank_of_group)) if int(rank_of_group[k]) == rank]


def allreduce_grads(grad, world, group=None):
    """The one data-path collective: sum of the flat gradient buffer over the ranks.  Without an
    initialised process group (bench.py --world-sim: one process plays each rank in turn) there
    is nothing to reduce with."""
    if world > 1 and torch.distributed.is_available() and torch.distributed.is_initialized():
        torch.distributed.all_reduce(grad, group=group)


class DeviceGraph:
    """CSR graph resident in HBM (+ the node_map workspace the relabel kernels use)."""

    def __init__(self, row_ptr, col, device="cuda"):
        if torch.is_tensor(row_ptr):
            self.row_ptr = row_ptr.to(device=device, dtype=torch.int64).contiguous()
            self.col = col.to(device=device, dtype=torch.int32).contiguous()
        else:
            self.row_ptr = torch.as_tensor(np.asarray(row_ptr, np.int64)).to(device)
            self.col = torch.as_tensor(np.asarray(col, np.int32)).to(device)
        self.N = self.row_ptr.numel() - 1
        self.ws = torch.empty(B.graph_workspace_bytes(self.N), dtype=torch.uint8, device=device)
        self.g = B.Graph()
        self.g.num_nodes = self.N
        self.g.nnz = self.col.numel()
        self.g.row_ptr = self.row_ptr.data_ptr()
        self.g.col = self.col.data_ptr()
        B.graph_prepare(self.g, self.ws)
        self._sched_ws = None
        self._g_sched = None

    @property
    def g_sched(self):
        """A second view of the graph with its own node_map / bitmap workspace, for a scheduler
        that runs on another stream while the blocks of the current epoch are built."""
        if self._g_sched is None:
            self._sched_ws = torch.empty_like(self.ws)
            self._g_sched = B.Graph()
            self._g_sched.num_nodes, self._g_sched.nnz = self.g.num_nodes, self.g.nnz
            self._g_sched.row_ptr, self._g_sched.col = self.g.row_ptr, self.g.col
            B.graph_prepare(self._g_sched, self._sched_ws)
        return self._g_sched


class PlanBuffers:
    """One set of buffalo_bucketize outputs (device arrays + host arrays + the Plan struct)."""

    def __init__(self, S, k_max, F, L, device):
        self.group_of_seed = torch.empty(S, dtype=torch.int32, device=device)
        self.group_seeds = torch.empty(S, dtype=torch.int32, device=device)
        self.group_offsets = torch.empty(k_max + 1, dtype=torch.int64, device=device)
        self.offs_h = np.zeros(k_max + 1, np.int64)
        self.est_h = np.zeros(k_max, np.int64)
        self.rank_h = np.zeros(k_max, np.int32)
        self.hist_h = np.zeros(F + 1, np.int64)
        self.sizes_h = np.zeros((k_max, 2 * L + 1), np.int64)     # exact per-group block sizes
        self.plan = B.Plan()
        self.plan.group_of_seed = self.group_of_seed.data_ptr()
        self.plan.group_seeds = self.group_seeds.data_ptr()
        self.plan.group_offsets = self.group_offsets.data_ptr()
        self.plan.group_offsets_h = self.offs_h.ctypes.data
        self.plan.est_bytes_h = self.est_h.ctypes.data
        self.plan.rank_of_group_h = self.rank_h.ctypes.data
        self.plan.hist_h = self.hist_h.ctypes.data
        self.plan.group_sizes_h = self.sizes_h.ctypes.data


class ShardedFeatures:
    """A node-id-range sharded bf16 feature table (include/buffalo.h buffalo_feature_shards; the
    IGB-shaped configuration): shard k holds the rows [k * rows_per_shard, ...).
    `shards` are CUDA tensors of this process (its own shard, or all of them on one GPU) or raw
    device pointers opened from peers (buffalo_ipc_open); `pitch` is the row pitch in elements."""

    def __init__(self, shards, rows_per_shard, num_rows, pitch, keep=()):
        self.struct = B.make_shards(shards, rows_per_shard)
        self.rows_per_shard = int(rows_per_shard)
        self.shape = (int(num_rows), int(pitch))
        self.dtype = torch.bfloat16
        self._keep = list(shards) + list(keep)
        local = [s for s in shards if torch.is_tensor(s)]
        self.first = local[0] if local else None        # a local tensor for the binding's dtype check


def exchange_shards(local, rank, world, rows_per_shard, num_rows, group=None):
    """One process per GPU: export this rank's shard (a CUDA tensor), all-gather the 64-byte IPC
    handles over the process group, open the peers' shards (NVLink peer mappings on an NVSwitch
    box).  Returns (ShardedFeatures, close) — call close() before the peers free their shards."""
    import torch.distributed as dist
    handles = [None] * world
    dist.all_gather_object(handles, B.ipc_export(local), group=group)
    ptrs, opened = [], []
    for r in range(world):
        if r == rank:
            ptrs.append(local)
        else:
            p = B.ipc_open(handles[r])
            opened.append((handles[r], p))
            ptrs.append(p)

    def close():
        for h, p in opened:
            B.ipc_close(h, p)
        opened.clear()
    return ShardedFeatures(ptrs, rows_per_shard, num_rows, local.shape[1], keep=[local]), close


class SageParams:
    """fp32 master weights/biases (Xavier init from synth), flat gradient buffer, packed copies.
    The flat buffers are layer-major: layer l's W, b and aggregator weights (pool W_pool, b_pool;
    LSTM W_ih, W_hh, b; GAT a_l, a_r) form one contiguous slice (layer_slice[l - 1]), so a
    layer's gradient can be all-reduced as soon as its last backward has run."""

    def __init__(self, model, Ws, bs, device="cuda", Wps=None, bps=None, lstm=None, gat=None):
        self.model = model
        self.L = L = model.num_layers
        Wps, bps = list(Wps or []), list(bps or [])
        Wih, Whh, bl = [list(x) for x in lstm] if lstm else ([], [], [])
        als, ars = [list(x) for x in gat] if gat else ([], [])
        per_layer = []
        for l in range(L):
            items = [("W", Ws[l]), ("b", bs[l])]                  # (name, array) in slice order
            if Wps:
                items += [("Wp", Wps[l]), ("bp", bps[l])]
            if Wih:
                items += [("Wih", Wih[l]), ("Whh", Whh[l]), ("bl", bl[l])]
            if als:
                items += [("al", als[l]), ("ar", ars[l])]
            per_layer.append(items)
        total = sum(int(np.asarray(a).size) for items in per_layer for _, a in items)
        self.flat = torch.zeros(total, dtype=torch.float32, device=device)
        self.grad = torch.zeros_like(self.flat)
        views = {k: ([], []) for k in ("W", "b", "Wp", "bp", "Wih", "Whh", "bl", "al", "ar")}
        self.layer_slice = []
        off = 0
        for items in per_layer:
            start = off
            for name, a in items:
                a = np.asarray(a)
                p = self.flat[off:off + a.size].view(a.shape)
                p.copy_(torch.as_tensor(a))
                views[name][0].append(p)
                views[name][1].append(self.grad[off:off + a.size].view(a.shape))
                off += a.size
            self.layer_slice.append((start, off))
        self.W, self.dW = views["W"]
        self.b, self.db = views["b"]
        # GraphSAGE-pool weights (R28), in the same flat buffers (one allreduce, one SGD step)
        self.Wp, self.dWp = views["Wp"]
        self.bp, self.dbp = views["bp"]
        # GraphSAGE-LSTM weights (R29): W_ih, W_hh [4d, d], b [4d] per layer
        self.lstm = [views["Wih"][0], views["Whh"][0], views["bl"][0]]
        self.dlstm = [views["Wih"][1], views["Whh"][1], views["bl"][1]]
        # GAT attention vectors (R30): a_l, a_r [d_l] per layer
        self.al, self.dal = views["al"]
        self.ar, self.dar = views["ar"]
        self.is_gat = model.aggregator == B.AGG_GAT      # GAT's W_l is [d_l, d_{l-1}]: no packed Update copy
        self.packed = [None if self.is_gat else
                       torch.empty(B.packed_weight_bytes(model, l), dtype=torch.uint8, device=device)
                       for l in range(1, self.L + 1)]
        self.repack()

    def repack(self):
        if self.is_gat:
            return
        for l in range(1, self.L + 1):
            B.pack_weights(self.model, l, self.W[l - 1], self.packed[l - 1])


class Trainer:
    def __init__(self, graph, feats, labels, seeds, dims, fanout, F, Ws, bs, feat_dtype=B.FP32,
                 gemm_mode=B.GEMM_FFMA, mem_budget=(1 << 63) - 1, C_ppm=0, k_min=1, k_max=4096,
                 base_seed=3, rank=0, world=1, process_group=None, device="cuda", aggregator=B.AGG_MEAN,
                 Wps=None, bps=None, lstm=None, gat=None, pipeline=False, sample_cache=True, k_multiple=1,
                 share_stats=True, allgather=None):
        self.graph = graph if isinstance(graph, DeviceGraph) else DeviceGraph(*graph, device=device)
        self.feats = feats
        self.labels = labels
        if not (seeds.is_cuda and seeds.dtype == torch.int32 and labels.dtype == torch.int32):
            raise TypeError("seeds and labels must be int32 CUDA tensors")
        self._seeds = [seeds]
        self._seeds_version = 0
        self.S = seeds.numel()
        self.dims = list(dims)
        self.L = len(dims) - 1
        self.fanout = list(fanout)
        self.F = F
        self.base_seed = base_seed
        self.pool = aggregator == B.AGG_POOL
        self.is_lstm = aggregator == B.AGG_LSTM
        if self.pool and Wps is None:
            raise ValueError("the pool aggregator needs its weights (Wps, bps)")
        self.is_gat = aggregator == B.AGG_GAT
        if self.is_gat and gat is None:
            raise ValueError("GAT needs its attention vectors (a_l, a_r per layer)")
        if self.is_lstm and lstm is None:
            raise ValueError("the LSTM aggregator needs its weights (W_ih, W_hh, b per layer)")
        self.sharded = isinstance(feats, ShardedFeatures)
        self.model = B.make_model(dims, feat_dtype, gemm_mode, feats.shape[1], aggregator,
                                  shards=feats.struct if self.sharded else None)
        # with a process group, the K loop's micro-bucket statistics are shared out over the ranks
        # (buffalo_sched.allgather); every rank still derives the identical plan
        # (allgather: an explicit buffalo_sched.allgather callback instead, e.g. bench.py's world-sim
        # replay of the all-gathers of N simulated ranks)
        ag = allgather if (share_stats and world > 1) else None
        if ag is None and share_stats and world > 1 and torch.distributed.is_available() and \
                torch.distributed.is_initialized():
            nccl = torch.distributed.get_backend(process_group) == "nccl"
            ag = B.make_allgather(world, process_group, torch.device(device) if nccl else None)
        self.sched = B.make_sched(mem_budget, C_ppm, k_min, k_max, world, k_multiple, rank, ag)
        self.params = SageParams(self.model, Ws, bs, device, Wps, bps, lstm, gat)
        self.rank, self.world, self.pg = rank, world, process_group
        self.device = device
        # scheduler outputs: two buffer sets, so that with pipeline=True the plan of epoch e+1 is
        # computed (on a side stream, with its own graph workspace) while epoch e trains from the
        # other set.  The plan is a function of (seeds, epoch) only, never of the weights.
        self.k_cap = k_max
        self._pb = [PlanBuffers(self.S, k_max, F, self.L, device)]
        self._cur = 0
        self.pipeline = pipeline
        self._ahead = None
        if pipeline:
            self._pb.append(PlanBuffers(self.S, k_max, F, self.L, device))
            self._seeds.append(torch.empty_like(seeds))       # the seed batch the ahead plan is for
            self._side = torch.cuda.Stream(device=device)
        # sample cache per plan-buffer set (include/buffalo.h): the scheduler's first statistics
        # pass stores every sampled neighbour list of the batch, the build copies them
        N = self.graph.N
        if self.sched.allgather:
            sample_cache = False             # shared statistics: the scheduler fills no cache
        self._cache = [[torch.empty(N * f, dtype=torch.int32, device=device) if (sample_cache and f > 0) else None
                        for f in self.fanout] for _ in self._pb]
        self._cache_epoch = [None] * len(self._pb)
        sampler = B.make_sampler(self.fanout, F, base_seed)
        wsb = B.bucketize_workspace_bytes(self.graph.g, self.S, sampler, self.model)
        self.bucket_ws = torch.empty(wsb, dtype=torch.uint8, device=device)
        self.arena = torch.empty(0, dtype=torch.uint8, device=device)
        self.loss = torch.zeros(1, dtype=torch.float32, device=device)
        self.blocks = B.Blocks()
        self.last = {}

    # plan of the current epoch (the buffer set in use) and the seed batch it was made for
    seeds = property(lambda self: self._seeds[self._cur])
    group_of_seed = property(lambda self: self._pb[self._cur].group_of_seed)
    group_seeds = property(lambda self: self._pb[self._cur].group_seeds)
    group_offsets = property(lambda self: self._pb[self._cur].group_offsets)
    offs_h = property(lambda self: self._pb[self._cur].offs_h)
    est_h = property(lambda self: self._pb[self._cur].est_h)
    rank_h = property(lambda self: self._pb[self._cur].rank_h)
    hist_h = property(lambda self: self._pb[self._cur].hist_h)
    sizes_h = property(lambda self: self._pb[self._cur].sizes_h)
    plan = property(lambda self: self._pb[self._cur].plan)

    # --------------------------------------------------------------- pieces of Alg. 2
    def sampler(self, epoch):
        """The sampler of `epoch`; it carries the current buffer set's sample cache when that
        cache was filled by the scheduler for this epoch."""
        cache = self._cache[self._cur] if self._cache_epoch[self._cur] == epoch else None
        return B.make_sampler(self.fanout, self.F, self.base_seed + epoch, cache)

    def schedule(self, epoch):
        """Alg. 3 for `epoch` into the current plan buffers (stream-ordered on the current stream)."""
        self._ahead = None
        return self._schedule_into(self._cur, epoch, self.graph.g)

    def set_seeds(self, seeds):
        """Replaces the seed batch (a device or pinned host int32 tensor of the same size).  A plan
        computed ahead for the old batch is dropped, so the next epoch schedules the new one."""
        if seeds.numel() != self.S or seeds.dtype != torch.int32:
            raise ValueError("set_seeds: expected int32 seeds of the trainer's batch size")
        self.seeds.copy_(seeds, non_blocking=True)
        self._seeds_version += 1
        self._ahead = None

    def fixed_bytes(self):
        """Device bytes the trainer holds outside the micro-batch arena (graph workspaces,
        scheduler workspace, plan buffers, sample caches, seeds, parameters and gradients)."""
        ts = [self.graph.ws, self.graph._sched_ws, self.bucket_ws, self.loss, self.params.flat, self.params.grad]
        ts += [t for t in self._seeds] + [p for p in self.params.packed if p is not None]
        ts += [c for cs in self._cache for c in cs if c is not None]
        ts += [t for pb in self._pb for t in (pb.group_of_seed, pb.group_seeds, pb.group_offsets)]
        return int(sum(t.numel() * t.element_size() for t in ts if t is not None))

    def _schedule_into(self, buf, epoch, g):
        pb = self._pb[buf]
        self._cache_epoch[buf] = None
        sp = B.make_sampler(self.fanout, self.F, self.base_seed + epoch, self._cache[buf])
        B.bucketize(g, self._seeds[buf], sp, self.model, self.sched, pb.plan, self.bucket_ws)
        self._cache_epoch[buf] = epoch
        K = pb.plan.k_out
        return K, pb.offs_h[:K + 1].copy(), pb.est_h[:K].copy(), pb.rank_h[:K].copy()

    def _ensure_arena(self, nbytes):
        """Grows the micro-batch arena (with 1/8 headroom, so that the need drifting between
        epochs does not reallocate it every time)."""
        if self.arena.numel() < nbytes:
            self.arena = None
            self.arena = torch.empty(int(nbytes + nbytes // 8), dtype=torch.uint8, device=self.device)

    def build(self, off, n, sampler, sizes=None):
        """Blocks of the group at group_seeds[off:off+n]; sizes = its row of the plan's exact
        block sizes (sync-free build) or None (sizes read back while building)."""
        while True:
            try:
                return B.build_blocks(self.graph.g, self.group_seeds.data_ptr() + 4 * int(off), n, sampler,
                                      self.model, self.blocks, self.arena, sizes)
            except B.BuffaloError as e:
                if e.status != B.ERR_CAPACITY:
                    raise
                self._ensure_arena(max(int(e.required * 1.25), 2 * self.arena.numel(), 1 << 20))

    def _feat_arg(self):
        """Layer-1 h_src: the feature table (ignored by the library for a sharded one)."""
        return self.feats.first if self.sharded else self.feats

    def forward(self):
        m, p, blks = self.model, self.params, self.blocks
        h, ld = self._feat_arg(), self.feats.shape[1]
        for l in range(1, self.L + 1):
            b = blks.layer[l - 1]
            if self.is_gat:
                B.gat_fwd(b, l, m, h, ld, p.W[l - 1], p.al[l - 1], p.ar[l - 1], p.b[l - 1], b.out, b.ld_out)
            elif self.is_lstm:
                B.lstm_fwd(b, l, m, h, ld, p.lstm[0][l - 1], p.lstm[1][l - 1], p.lstm[2][l - 1], p.W[l - 1],
                           p.packed[l - 1], p.b[l - 1], b.out, b.ld_out, b.agg, b.ld_agg)
            elif self.pool:
                B.pool_fwd(b, l, m, h, ld, p.Wp[l - 1], p.bp[l - 1], p.W[l - 1], p.packed[l - 1], p.b[l - 1],
                           b.out, b.ld_out, b.agg, b.ld_agg, b.pool_P, b.pool_arg, b.ld_pool)
            else:
                B.sage_fwd(b, l, m, h, ld, p.W[l - 1], p.packed[l - 1], p.b[l - 1], b.out, b.ld_out, b.agg,
                           b.ld_agg)
            h, ld = b.out, b.ld_out

    def backward(self, after_layer=None):
        """Alg. 2 l.11-12 for layers L..1; after_layer(l), if given, runs once layer l's backward
        is enqueued (the last group's hook starts that layer's gradient all-reduce)."""
        for l in range(self.L, 0, -1):
            self._backward_layer(l)
            if after_layer is not None:
                after_layer(l)

    def _backward_layer(self, l):
        m, p, blks = self.model, self.params, self.blocks
        if True:
            b = blks.layer[l - 1]
            if l > 1:
                prev = blks.layer[l - 2]
                h_src, ld_src, dh_src, ld_dh_src = prev.out, prev.ld_out, prev.dh, prev.ld_dh
            else:
                h_src, ld_src, dh_src, ld_dh_src = self._feat_arg(), self.feats.shape[1], None, 0
            h_dst = b.out if l < self.L else None
            if self.is_gat:
                B.gat_bwd(b, l, m, b.dh, b.ld_dh, h_src, ld_src, h_dst, b.ld_out, p.W[l - 1], p.al[l - 1],
                          p.ar[l - 1], p.dW[l - 1], p.db[l - 1], p.dal[l - 1], p.dar[l - 1], dh_src, ld_dh_src,
                          b.bwd_scratch, b.bwd_scratch_bytes)
                return
            if self.is_lstm:
                B.lstm_bwd(b, l, m, b.dh, b.ld_dh, h_src, ld_src, b.agg, b.ld_agg, h_dst, b.ld_out,
                           p.lstm[0][l - 1], p.lstm[1][l - 1], p.W[l - 1], p.dlstm[0][l - 1], p.dlstm[1][l - 1],
                           p.dlstm[2][l - 1], p.dW[l - 1], p.db[l - 1], dh_src, ld_dh_src, b.bwd_scratch,
                           b.bwd_scratch_bytes)
                return
            if self.pool:
                B.pool_bwd(b, l, m, b.dh, b.ld_dh, h_src, ld_src, b.agg, b.ld_agg, h_dst, b.ld_out, b.pool_P,
                           b.pool_arg, b.ld_pool, p.Wp[l - 1], p.W[l - 1], p.dWp[l - 1], p.dbp[l - 1],
                           p.dW[l - 1], p.db[l - 1], dh_src, ld_dh_src, b.bwd_scratch, b.bwd_scratch_bytes)
                return
            B.sage_bwd(b, l, m, b.dh, b.ld_dh, h_src, ld_src, b.agg, b.ld_agg, h_dst, b.ld_out,
                       p.W[l - 1], p.packed[l - 1], p.dW[l - 1], p.db[l - 1], dh_src, ld_dh_src,
                       b.bwd_scratch, b.bwd_scratch_bytes)

    def loss_and_grad(self, off, n):
        b = self.blocks.layer[self.L - 1]
        ids = self.group_seeds.data_ptr() + 4 * int(off)
        B.softmax_ce(b.out, b.ld_out, n, self.dims[-1], self.labels, ids, self.S, self.loss, b.dh, b.ld_dh)

    def microbatch(self, off, n, sampler, sizes=None, after_layer=None):
        self.build(off, n, sampler, sizes)
        self.forward()
        self.loss_and_grad(off, n)
        self.backward(after_layer)
        blk = self.blocks
        return dict(edges=sum(blk.layer[l].n_edges for l in range(self.L)),
                    n=[blk.layer[0].n_src] + [blk.layer[l].n_dst for l in range(self.L)],
                    e=[blk.layer[l].n_edges for l in range(self.L)],
                    peak=blk.arena_peak, est_lo=blk.est_lo, est_hi=blk.est_hi)

    # a 4-byte word no kernel writes: a NaN payload in fp32, a NaN high half in bf16, and an int32
    # above every node id / offset of a micro-batch
    HW_SENTINEL = 0x7FBADF00

    def measure_high_water(self, k, epoch, guard=1 << 20):
        """Measured arena high-water mark of group k (independent of the memory model): the arena
        is filled with HW_SENTINEL, the library is handed exactly lo = buffalo_estimate_mem's
        exact need of the group, and after build + forward + loss + backward the highest word
        that no longer holds the sentinel gives the bytes actually touched (a `guard` of sentinel
        words past lo must stay intact).  Accumulates into the gradients like microbatch().
        Returns (high_water_bytes, lo, hi, guard_intact)."""
        L = self.L
        sizes = self.sizes_h[k]
        lo, hi = B.estimate_mem(sizes[:L + 1], sizes[L + 1:], self.model)
        total = (lo + guard + 255) // 256 * 256
        self._ensure_arena(total)
        keep = self.arena
        words = keep[:total].view(torch.int32)
        words.fill_(self.HW_SENTINEL)
        self.arena = keep[:lo]
        try:
            offs = self.offs_h
            self.microbatch(int(offs[k]), int(offs[k + 1] - offs[k]), self.sampler(epoch), sizes)
        finally:
            self.arena = keep
        torch.cuda.synchronize()
        changed = words != self.HW_SENTINEL
        CH = 1 << 16
        full = changed.numel() // CH * CH
        last = -1
        if changed.numel() > full and bool(changed[full:].any()):
            last = full + int(torch.nonzero(changed[full:]).max())
        elif full:
            hit = torch.nonzero(changed[:full].view(-1, CH).any(dim=1))
            if hit.numel():
                c = int(hit.max())
                last = c * CH + int(torch.nonzero(changed[c * CH:(c + 1) * CH]).max())
        hw = 4 * (last + 1)
        guard_ok = not bool(changed[(lo + 3) // 4:].any())
        del changed
        return hw, lo, hi, guard_ok

    def _overlap_stream(self):
        """The communication stream of the per-layer gradient all-reduce (N > 1 with an
        initialised process group), else None (one all-reduce after the last group)."""
        if not (self.world > 1 and torch.distributed.is_available() and torch.distributed.is_initialized()):
            return None
        if getattr(self, "_comm", None) is None:
            self._comm = torch.cuda.Stream(device=self.device)
        return self._comm

    def allreduce(self):
        allreduce_grads(self.params.grad, self.world, self.pg)

    def step(self, lr):
        B.sgd_step(self.params.flat, self.params.grad, lr)
        self.params.repack()

    def run_epoch(self, epoch=0, lr=0.01, timers=False, next_seeds=None):
        """One Buffalo iteration; returns stats (K, own groups, aggregated edges, ...).
        pipeline=True: the plan was computed during the previous call (if it was for this epoch
        and the seed batch has not been replaced since), and the next epoch's plan is computed on
        the side stream while this epoch's work runs — for `next_seeds` (a pinned host or device
        int32 tensor, copied on the side stream) if given, else for the current batch."""
        main = torch.cuda.current_stream()
        a = self._ahead
        self._ahead = None
        if self.pipeline and a is not None and a["epoch"] == epoch and a["version"] == self._seeds_version:
            self._cur = a["buf"]
            main.wait_event(a["done"])
            K, offs, est, ranks = a["K"], a["offs"], a["est"], a["ranks"]
        else:
            K, offs, est, ranks = self._schedule_into(self._cur, epoch, self.graph.g)
        before = main.record_event()        # the next plan depends on nothing enqueued after this
        self.loss.zero_()
        mine = own_groups(ranks, self.rank)
        L = self.L
        need = [B.estimate_mem(self.sizes_h[k, :L + 1], self.sizes_h[k, L + 1:], self.model)[0] for k in mine]
        self._ensure_arena(max(need) if need else 1 << 20)          # exact (R15): no build retries
        sampler = self.sampler(epoch)
        groups = []
        comm = self._overlap_stream()
        pending = []

        def reduce_layer(l):
            # the last own group's layer-l backward is enqueued: layer l's gradient slice is final
            # on this rank, so its all-reduce (NCCL, comm stream) overlaps layers l-1..1
            a, b_ = self.params.layer_slice[l - 1]
            ev = torch.cuda.current_stream().record_event()
            comm.wait_event(ev)
            with torch.cuda.stream(comm):
                allreduce_grads(self.params.grad[a:b_], self.world, self.pg)
            pending.append(l)

        for i, k in enumerate(mine):
            hook = reduce_layer if (comm is not None and i == len(mine) - 1) else None
            groups.append(dict(self.microbatch(offs[k], int(offs[k + 1] - offs[k]), sampler, self.sizes_h[k],
                                               hook), k=k))
        if comm is None:
            self.allreduce()
        else:
            if not mine:                                   # no own group: contribute zeros
                for l in range(self.L, 0, -1):
                    reduce_layer(l)
            torch.cuda.current_stream().wait_stream(comm)
        self.step(lr)
        self.last = dict(K=K, k_tried=self.plan.k_tried, exploded=self.plan.exploded, est=est,
                         ranks=ranks, groups=groups, edges=sum(g["edges"] for g in groups),
                         hist=self.hist_h.copy())
        if self.pipeline:
            # Alg. 3 of epoch + 1 on the side stream (own graph workspace, the other plan buffers),
            # overlapping this epoch's build / forward / backward on the main stream
            nb = 1 - self._cur
            self._side.wait_event(before)
            with torch.cuda.stream(self._side):
                if next_seeds is not None:
                    if next_seeds.numel() != self.S or next_seeds.dtype != torch.int32:
                        raise ValueError("next_seeds: expected int32 seeds of the trainer's batch size")
                    self._seeds[nb].copy_(next_seeds, non_blocking=True)
                    self._seeds_version += 1
                else:
                    self._seeds[nb].copy_(self._seeds[self._cur])
                Kn, offn, estn, rankn = self._schedule_into(nb, epoch + 1, self.graph.g_sched)
                done = self._side.record_event()
            self._ahead = dict(epoch=epoch + 1, buf=nb, K=Kn, offs=offn, est=estn, ranks=rankn, done=done,
                               version=self._seeds_version)
        return self.last
