#!/usr/bin/env python
"""Benchmark of Buffalo's data-parallel hot path on B200 (BASELINE.json metric:
"epoch time & aggregated edges/s under fixed mem budget at 1/2/4/8 B200").

A step = one Buffalo iteration (Alg. 2) over the whole seed batch:
bucketize (Alg. 3/4 + Eq. 1-2) + for every own bucket group: block generation, L fused
SAGE-mean forward layers, loss, L backward layers + NCCL gradient allreduce (N > 1) + SGD.
value = aggregated block edges of all ranks / max-over-ranks device time (edges/s).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config products|arxiv|cora]

The default workload is BASELINE.json configs[2] (products-shaped, fixed memory budget, the
config the metric is quoted on at 1/2/4/8 GPUs); arxiv and Cora are selectable.
                  [--gemm bf16|ffma] [--impl ours|reference]

Under torchrun (N > 1) every rank runs its own groups (k_min = N, LPT by estimate).
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth.graphs import CONFIGS, features, labels, random_graph, seed_nodes, xavier_weights  # noqa: E402

WORKLOADS = {
    "arxiv": ("ogbn-arxiv-shaped power-law graph (169,343 nodes, 1,166,243 undirected edges, 128-d), "
              "3-layer SAGE-mean 128-256-256-40, full-neighbour blocks, F=10, 90,941 seeds, K=4 bucket groups"),
    "cora": ("Cora-sized synthetic graph (2,708 nodes, 5,278 edges, 1,433-d), 2-layer SAGE-mean "
             "1433-256-7, fanout (10,25), 4 partitions"),
    "arxiv_lstm": ("ogbn-arxiv-shaped power-law graph (169,343 nodes, 1,166,243 undirected edges, 128-d), "
                   "2-layer SAGE-LSTM 128-128-40 (LSTM hidden 128, PAPER.md:351), fanout (10,25), F=25, "
                   "90,941 seeds, budget forcing >= 2 bucket groups"),
    "papers": ("ogbn-papers100M-shaped power-law graph (111,059,956 nodes, 1,615,685,872 undirected edges, "
               "128-d), 2-layer SAGE-mean 128-256-172, fanout (10,25), F=25, 1,207,179 seeds, budget forcing >= 8 "
               "bucket groups"),
    "products": ("ogbn-products-shaped power-law graph (2,449,029 nodes, 61,859,140 edges, 100-d), 3-layer "
                 "SAGE-mean 100-256-256-47, fanout (10,25,30), budget forcing >= 8 bucket groups"),
    "igb_small": ("IGB-large-shaped power-law graph at 1/8 scale (12,500,000 nodes, 150,000,000 undirected edges, "
                  "1024-d bf16 features = 25.6 GB held as node-range shards: 8 on one GPU, one per rank over "
                  "CUDA IPC / NVLink at N > 1), 3-layer SAGE-mean 1024-256-256-19, fanout (5,10,15), F=15, "
                  "125,000 seeds, budget forcing >= 8 bucket groups"),
    "igb": ("IGB-large-shaped power-law graph (100,000,000 nodes, 1,200,000,000 undirected edges, 1024-d bf16 "
            "features = 205 GB sharded by node range, one shard per rank over CUDA IPC / NVLink), 3-layer "
            "SAGE-mean 1024-256-256-19, fanout (5,10,15), F=15, 1,000,000 seeds, budget forcing >= 8 groups"),
}
SHARDED = ("igb", "igb_small")


# Table II's average clustering coefficients, logged beside the C measured
# on the synthetic graph (reading R27; the Chung-Lu graphs have far fewer triangles)
C_TABLE2 = {"cora": 0.24, "arxiv": 0.226, "arxiv_lstm": 0.226, "products": 0.411, "papers": 0.085}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="products", choices=list(WORKLOADS))
    ap.add_argument("--gemm", default="bf16", choices=["bf16", "ffma"])
    ap.add_argument("--aggregator", default="mean", choices=["mean", "pool", "lstm", "gat"],
                    help="pool / lstm: GraphSAGE-pool / -LSTM, gat: GAT (SURVEY §8(f) NEXT 2 / 1 / 3), fp32 FFMA "
                         "path only")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--cpu-baseline-seconds", type=float, default=20.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--world-sim", type=int, default=0,
                    help="one GPU plays each of N ranks in turn (plan for N GPUs, per-rank epoch times)")
    ap.add_argument("--sim-shared", action="store_true",
                    help="with --world-sim N: the ranks share the scheduler's statistics passes "
                         "(buffalo_sched.allgather) — the all-gathers of the N ranks are recorded untimed, "
                         "then each rank's timed epochs measure only its own share and replay the rest")
    ap.add_argument("--rank-balanced-k", action="store_true",
                    help="reading R31: only K that are multiples of the GPU count (rank-aware grouping)")
    ap.add_argument("--no-pipeline", action="store_true",
                    help="schedule each epoch synchronously (default: the next epoch's plan is computed on a "
                         "side stream while the current epoch trains)")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def make_inputs_device(cfg, feat_dtype=None, shards=None):
    """The same inputs as make_inputs, generated on the GPU by synth.device (bit-identical to
    the numpy recipe; a products-shaped graph takes seconds instead of minutes on one core).
    feat_dtype: generate the feature table directly in that dtype (k/128 values are exact in
    bf16; the papers-shaped table is 28 GB in bf16, 57 GB in fp32).  shards: a list of node
    ranges (r0, r1): X is then the list of those row ranges of the table (separate allocations)."""
    import torch
    from synth import device as SD
    rp, col = SD.random_graph(cfg.N, cfg.pairs, cfg.kind)
    torch.cuda.empty_cache()
    pitch = ((cfg.d0 + 31) // 32) * 32
    if shards is not None:
        X = [SD.features_range(r0, r1, cfg.d0, pitch, dtype=feat_dtype or torch.float32) for r0, r1 in shards]
    else:
        X = SD.features(cfg.N, cfg.d0, pitch, dtype=feat_dtype or torch.float32)
    y = SD.labels(cfg.N, cfg.classes)
    seeds = SD.seed_nodes(cfg.N, cfg.S)
    Ws, bs = xavier_weights(cfg.dims)
    torch.cuda.synchronize()
    return rp, col, X, y, seeds, Ws, bs


def host_copies(*ts):
    return [t.cpu().numpy() if hasattr(t, "cpu") else t for t in ts]


def make_inputs(cfg):
    rp, col = random_graph(cfg.N, cfg.pairs, cfg.kind)
    # feature rows padded to a multiple of 64 B (32 bf16): a random row then costs whole 64-B
    # DRAM atoms only (measured +9% gather bandwidth for 200-B rows)
    X = features(cfg.N, cfg.d0, ((cfg.d0 + 31) // 32) * 32)
    y = labels(cfg.N, cfg.classes)
    seeds = seed_nodes(cfg.N, cfg.S)
    Ws, bs = xavier_weights(cfg.dims)
    return rp, col, X, y, seeds, Ws, bs


# ----------------------------------------------------------------------------- oracle arm
def oracle_sample(cfg, rp, col, X, y, seeds, Ws, bs, seconds, edges_per_epoch=None):
    """The CPU oracle (oracle/, as it stands) on a bounded sample of the workload: one
    micro-batch of a contiguous slice of the seed batch, grown until ~`seconds` of work.  The
    oracle is single-threaded C (blocks) plus numpy/scipy (layer math); BLAS is pinned to one
    thread so `cores` = 1 is what it used.  Its epoch time is extrapolated from the measured
    rate (aggregated edges of our epoch / oracle edges per second)."""
    import oracle as O
    from threadpoolctl import threadpool_limits
    g = O.Graph(rp, col)
    frac = 64
    n_edges, elapsed, used = 0, 0.0, 0
    with threadpool_limits(limits=1):
        while True:
            part = seeds[: max(1, len(seeds) // frac)]
            t = time.perf_counter()
            loss, grads, blocks = O.microbatch_step(g, part, X[:, :cfg.d0], y, Ws, bs, cfg.L, cfg.fanout, 3,
                                                    len(seeds))
            dt = time.perf_counter() - t
            n_edges, elapsed, used = sum(b["n_edges"] for b in blocks), dt, len(part)
            if dt * 3 > seconds or frac == 1:
                break
            frac = max(1, frac // 4)
    rate = n_edges / elapsed
    out = dict(value=rate, unit="edges/s", cores=1, kind="oracle",
               sample=f"one micro-batch of {used} of {len(seeds)} seeds ({n_edges} block edges, "
                      f"{elapsed:.2f} s, measured): C block generation + float64 numpy/scipy SAGE fwd/bwd, "
                      f"1 thread (BLAS pinned)")
    if edges_per_epoch:
        out["epoch_s_extrapolated"] = edges_per_epoch / rate
    return out


def run_reference(args, cfg):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    if args.config in SHARDED:
        print(json.dumps({"impl": "reference", "unavailable": "the IGB-shaped 1024-d table (25.6-205 GB) is not "
                          "copied to the host for the oracle; its arm runs on the products/papers/arxiv configs"}))
        return
    try:
        import torch
        on_gpu = torch.cuda.is_available()
    except ImportError:
        on_gpu = False
    if on_gpu:       # same inputs, generated on the device (synth.device), then copied to the host
        rp, col, X, y, seeds, Ws, bs = make_inputs_device(cfg)
        rp, col, X, y, seeds = host_copies(rp, col, X, y, seeds)
    else:
        rp, col, X, y, seeds, Ws, bs = make_inputs(cfg)
    import oracle as O
    g = O.Graph(rp, col)
    # bounded sample per step (~1-5 s of oracle work; 35 steps end within a few minutes)
    part = seeds[: max(1, len(seeds) // {"products": 150, "cora": 1}.get(args.config, 16))]
    times, edges = [], 0
    for i in range(args.warmup + args.steps):
        t = time.perf_counter()
        _, _, blocks = O.microbatch_step(g, part, X[:, :cfg.d0], y, Ws, bs, cfg.L, cfg.fanout, 3 + i, len(seeds))
        dt = time.perf_counter() - t
        if i >= args.warmup:
            times.append(dt)
            edges += sum(b["n_edges"] for b in blocks)
    v = edges / sum(times)
    try:                     # the threads the oracle's BLAS calls used (the block builder is single-threaded C)
        from threadpoolctl import threadpool_info
        blas_threads = max([1] + [int(i.get("num_threads", 1)) for i in threadpool_info()])
    except Exception:        # noqa: BLE001
        blas_threads = 1
    line = dict(metric="aggregated edges/s (epoch of Buffalo hot path)", value=v, unit="edges/s",
                n_gpus=0, steps=args.steps, warmup=args.warmup, ms_per_step=1e3 * statistics.mean(times),
                higher_is_better=True, scaling="strong", vs_baseline=None, dtype="f64", data="synthetic",
                impl="reference",
                config={"workload": WORKLOADS[args.config], "sample": f"{len(part)} seeds per step"},
                cpu_baseline=dict(value=v, unit="edges/s", kind="oracle", cores=blas_threads,
                                  sample=f"per step one micro-batch of {len(part)} of {len(seeds)} seeds: C block "
                                         f"generation on 1 thread, float64 numpy/scipy layer math with BLAS on "
                                         f"{blas_threads} thread(s) ({len(os.sched_getaffinity(0))} host cores "
                                         f"available)"),
                e2e=dict(value=v, unit="edges/s", h2d_bytes_per_step=0, d2h_bytes_per_step=0))
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- clocks
class Clocks:
    """SM clock and throttle reasons sampled every 5 ms during the timed region (NVML in a
    thread; nvidia-smi -lms 20 if NVML is unavailable)."""
    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "hw_power_brake_slowdown": 0x80, "sw_power_cap": 0x4}

    def __init__(self, index):
        self.index = index
        self.samples, self.reasons, self.max_mhz = [], set(), 0.0
        self.thread = self.proc = None
        self.stop_flag = False

    def _poll(self, nv, h):
        while not self.stop_flag:
            try:
                self.samples.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                for name, bit in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def start(self):
        try:
            import threading
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
            self.thread = threading.Thread(target=self._poll, args=(nv, h), daemon=True)
            self.thread.start()
        except Exception:
            q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
            try:
                self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                              "-i", str(self.index), "-lms", "20"], stdout=subprocess.PIPE,
                                             stderr=subprocess.DEVNULL, text=True)
            except OSError:
                self.proc = None

    def stop(self):
        if self.thread is not None:
            self.stop_flag = True
            self.thread.join()
        elif self.proc is not None:
            self.proc.terminate()
            out, _ = self.proc.communicate()
            names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
            for ln in out.strip().splitlines():
                f = [x.strip() for x in ln.split(",")]
                try:
                    self.samples.append(float(f[0]))
                    self.max_mhz = max(self.max_mhz, float(f[1]))
                except (ValueError, IndexError):
                    continue
                for n, v in zip(names, f[2:6]):
                    if v.lower() == "active":
                        self.reasons.add(n)
        if not self.samples:
            return None
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ----------------------------------------------------------------------------- diagnostics
def phase_breakdown(tr, epoch):
    """One sequential epoch (outside the timed region) with CUDA events around each phase on the
    main stream: schedule (Alg. 3), and per group build / forward / loss / backward, summed; plus
    the block-build rates of SURVEY §8(d): sampled (block) edges per second of build time and a
    sector-based effective bandwidth (per edge: one 32-B sector for the cached sample row or CSR
    entry, two random 32-B sectors for the relabel's node bitmap and node map, 8 B of col_local /
    col_global writes, 8 B for the transpose; per dst row 16 B of row_ptr, 4 B of id)."""
    import torch
    from paper_conf_hpca_yangzl25_b200 import buffalo as B

    def ev():
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        return e
    torch.cuda.synchronize()
    e0 = ev()
    K, offs, est, ranks = tr.schedule(epoch)
    e1 = ev()
    L = tr.L
    mine = [k for k in range(K) if int(ranks[k]) == tr.rank]
    tr._ensure_arena(max(B.estimate_mem(tr.sizes_h[k, :L + 1], tr.sizes_h[k, L + 1:], tr.model)[0] for k in mine))
    sampler = tr.sampler(epoch)
    marks, edges, dsts = [], 0, 0
    tr.loss.zero_()
    for k in mine:
        n = int(offs[k + 1] - offs[k])
        a = ev()
        tr.build(offs[k], n, sampler, tr.sizes_h[k])
        b = ev()
        tr.forward()
        c = ev()
        tr.loss_and_grad(offs[k], n)
        d = ev()
        tr.backward()
        e = ev()
        marks.append((a, b, c, d, e))
        edges += int(sum(tr.sizes_h[k, L + 1:]))
        dsts += int(sum(tr.sizes_h[k, 1:L + 1]))
    torch.cuda.synchronize()
    tr.params.grad.zero_()
    ph = {"schedule": e0.elapsed_time(e1), "build": 0.0, "forward": 0.0, "loss": 0.0, "backward": 0.0}
    for a, b, c, d, e in marks:
        ph["build"] += a.elapsed_time(b)
        ph["forward"] += b.elapsed_time(c)
        ph["loss"] += c.elapsed_time(d)
        ph["backward"] += d.elapsed_time(e)
    sector_bytes = edges * (3 * 32 + 8 + 8) + dsts * 20
    build = {"ms": ph["build"], "sampled_edges": edges, "edges_per_s": edges / (ph["build"] / 1e3),
             "sector_gbs": sector_bytes / (ph["build"] / 1e3) / 1e9, "launches_note": "sync-free (plan sizes)"}
    return {k: round(v, 3) for k, v in ph.items()}, build


def measured_memory(tr, epoch):
    """Per own group of `epoch`: the measured arena high-water (sentinel fill, Trainer.
    measure_high_water: independent of the memory model and of the allocator's bookkeeping)
    against the exact model (lo, hi) and the Eq. 2 group estimate (Table III's
    estimate-vs-measured comparison, :477-497)."""
    K, offs, est, ranks = tr.schedule(epoch)
    rows = []
    for k in range(K):
        if int(ranks[k]) != tr.rank:
            continue
        hw, lo, hi, ok = tr.measure_high_water(k, epoch)
        rows.append((k, hw, lo, hi, int(est[k]), ok))
    tr.params.grad.zero_()
    hw = np.array([r[1] for r in rows], np.float64)
    eq2 = np.array([r[4] for r in rows], np.float64)
    return {"budget_bytes": int(tr.sched.mem_budget), "groups": len(rows),
            "measured_high_water_max_bytes": int(hw.max()), "measured_high_water_min_bytes": int(hw.min()),
            "measured_spread_max_over_min": float(hw.max() / hw.min()),
            "measured_within_exact_model": bool(all(r[1] <= r[2] <= r[3] and r[5] for r in rows)),
            "exact_lo_minus_measured_max_bytes": int(max(r[2] - r[1] for r in rows)),
            "eq2_over_measured_mean": float(np.mean(eq2 / hw - 1.0)),
            "eq2_over_measured_max": float(np.max(eq2 / hw - 1.0)),
            "eq2_over_measured_min": float(np.min(eq2 / hw - 1.0)),
            "max_measured_over_budget": float(hw.max() / tr.sched.mem_budget),
            "fixed_device_bytes_outside_arena": tr.fixed_bytes(),
            "method": "arena filled with a sentinel word, library given exactly lo bytes; high-water = highest "
                      "overwritten word after build+fwd+loss+bwd; a 1 MiB sentinel guard past lo stays intact",
            "note": "Eq. 2 with R = 1 (C of the synthetic graphs is ~5e-4) sums the items' own estimates, so it "
                    "over-estimates the nodes they share; fixed bytes (graph workspaces, scheduler workspace, "
                    "sample caches, plans, weights) are outside M_ctr"}


# ----------------------------------------------------------------------------- world-sim
class AllgatherReplay:
    """buffalo_sched.allgather for the world-sim with shared statistics (--sim-shared): serves
    recorded all-gather results (the concatenated rows of all N ranks) in call order, after
    checking that the calling rank's own rows equal the recorded ones (every rank's passes are
    deterministic).  In record mode (`record` set) the call past the known results stores the
    rank's rows and fails, which aborts that bucketize run."""

    def __init__(self, world):
        import ctypes
        from paper_conf_hpca_yangzl25_b200 import buffalo as B
        self.world, self.rank, self.results, self.i, self.record = world, 0, [], 0, None
        self._ct = ctypes
        self.fn = B.ALLGATHER_FN(self._call)

    def _call(self, ctx, send, recv, nbytes):
        ct = self._ct
        own = ct.string_at(send, nbytes)
        if self.i >= len(self.results):
            if self.record is not None:
                self.record[self.rank] = own
            return 1
        res = self.results[self.i]
        if len(res) != self.world * nbytes or res[self.rank * nbytes:(self.rank + 1) * nbytes] != own:
            return 1
        ct.memmove(recv, res, len(res))
        self.i += 1
        return 0


def record_allgathers(rep, run_rank):
    """The all-gather results of one deterministic computation run by each of rep.world ranks:
    call i's result is assembled from every rank's rows at call i, each rank replaying calls
    0..i-1 (run_rank(r) runs rank r's computation with rep.fn as its all-gather and returns
    whether it completed); repeated until the runs complete.  Returns the results in call order."""
    R = []
    while True:
        rows = [None] * rep.world
        for r in range(rep.world):
            rep.rank, rep.results, rep.i, rep.record = r, R, 0, rows
            run_rank(r)
        done = [x is None for x in rows]
        assert all(done) or not any(done), "simulated ranks disagree on the number of all-gathers"
        if all(done):
            rep.record = None
            return R
        R.append(b"".join(rows))


def record_shared_stats(tr, rep, epochs):
    """record_allgathers of the scheduler runs of `epochs` for the N simulated ranks (untimed),
    in the order a pipelined Trainer asks for them (one schedule per epoch, ascending)."""
    import torch
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import PlanBuffers
    pb = PlanBuffers(tr.S, tr.k_cap, tr.F, tr.L, tr.device)
    s = tr.sched
    out = []
    for e in epochs:
        def run_rank(r):
            sched = B.make_sched(s.mem_budget, s.C_ppm, s.k_min, s.k_max, rep.world, s.k_multiple, r, rep.fn)
            sp = B.make_sampler(tr.fanout, tr.F, tr.base_seed + e)
            try:
                B.bucketize(tr.graph.g_sched, tr._seeds[0], sp, tr.model, sched, pb.plan, tr.bucket_ws)
            except B.BuffaloError:
                pass
            torch.cuda.synchronize()
        out.extend(record_allgathers(rep, run_rank))
    return out


def run_world_sim(args, tr, sim, flush, stream):
    """--world-sim N on one GPU: the plan is made for N GPUs (k_min = N, LPT rank assignment,
    optionally rank-aware K), and this one process plays each rank r in turn — its replicated
    scheduler (the pipelined side stream, full Alg. 3 every epoch) plus its own groups — timing
    `steps` epochs per rank with CUDA events.  The N-GPU epoch is then bounded by the slowest
    rank (the NCCL allreduce of the 0.6-2.7 MB gradient, tens of microseconds over NVLink, is not
    simulated).  Prints one JSON line with "mode": "world_sim" (not the driver's bench line)."""
    import torch
    per = []
    rep = getattr(tr, "_sim_replay", None)
    recorded = None
    if rep is not None:
        t_rec = time.perf_counter()
        recorded = record_shared_stats(tr, rep, range(args.warmup + args.steps + 1))
        t_rec = time.perf_counter() - t_rec
    for r in range(sim):
        tr.rank = r
        tr.sched.rank = r                       # group sizes are measured for the own groups only
        tr._ahead = None
        if rep is not None:
            rep.rank, rep.results, rep.i = r, recorded, 0
        for i in range(args.warmup):
            tr.run_epoch(epoch=i, lr=0.01)
        torch.cuda.synchronize()
        ms, edges, groups, K = [], 0, 0, 0
        for i in range(args.steps):
            flush.zero_()
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            st = tr.run_epoch(epoch=args.warmup + i, lr=0.01)
            s1.record(stream)
            s1.synchronize()
            ms.append(s0.elapsed_time(s1))
            edges += st["edges"]
            groups = len(st["groups"])
            K = st["K"]
        per.append({"rank": r, "ms_per_step": sum(ms) / len(ms), "groups": groups,
                    "edges_per_epoch": edges / args.steps})
    worst = max(p["ms_per_step"] for p in per)
    total_edges = sum(p["edges_per_epoch"] for p in per)
    line = {"mode": "world_sim", "world_sim": sim, "config": args.config, "K": K,
            "rank_balanced_k": bool(args.rank_balanced_k), "per_rank": per,
            "projected_epoch_ms": worst, "projected_edges_per_s": total_edges / (worst / 1e3),
            "rank_spread_max_over_min": worst / min(p["ms_per_step"] for p in per),
            "shared_stats": rep is not None,
            "note": ("one B200 plays each rank in turn (" +
                     ("its share of the scheduler's statistics passes, the other ranks' rows replayed from an "
                      "untimed recording (all-gather latency not included), no sample cache"
                      if rep is not None else "replicated scheduler") +
                     " + own groups); NCCL allreduce not included; the projected N-GPU epoch is the slowest rank")}
    if rep is not None:
        line["allgathers_per_epoch"] = len(recorded) / (args.warmup + args.steps + 1)
        line["record_s"] = t_rec
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def run_ours(args, cfg):
    import torch
    rank, world, local = dist_env()
    # one process per GPU; BUFFALO_DIST_BACKEND=gloo (testing only) lets several ranks share a GPU
    backend = os.environ.get("BUFFALO_DIST_BACKEND", "nccl")
    dev = local % torch.cuda.device_count() if backend != "nccl" else local
    torch.cuda.set_device(dev)
    pg = None
    if world > 1:
        if backend == "nccl":
            torch.distributed.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            torch.distributed.init_process_group(backend)
        pg = torch.distributed.group.WORLD
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer

    B.lib()
    t_gen = time.perf_counter()
    big = cfg.N > 50_000_000 or args.config in SHARDED  # bf16 table generated directly, no fp32 copy
    sharded = args.config in SHARDED
    shard_ranges, rps = None, None
    if sharded:
        if args.gemm != "bf16" or args.aggregator != "mean":
            raise SystemExit("the sharded IGB-shaped configs run the bf16 SAGE-mean path")
        P = 8 if world == 1 else world            # one GPU: 8 local shards; else one shard per rank
        rps = (cfg.N + P - 1) // P
        mine = range(P) if world == 1 else [rank]
        shard_ranges = [(k * rps, min(cfg.N, (k + 1) * rps)) for k in mine]
    rp, col, X, y, seeds, Ws, bs = make_inputs_device(cfg, torch.bfloat16 if (big and args.gemm == "bf16") else None,
                                                      shard_ranges)
    t_gen = time.perf_counter() - t_gen
    shard_close = None
    if sharded:
        from paper_conf_hpca_yangzl25_b200.train import ShardedFeatures, exchange_shards
        if world == 1:
            X = ShardedFeatures(X, rps, cfg.N, X[0].shape[1])
        else:
            X, shard_close = exchange_shards(X[0], rank, world, rps, cfg.N, group=pg)
    pool = args.aggregator == "pool"
    lstm = args.aggregator == "lstm"
    gat = args.aggregator == "gat"
    if pool or lstm or gat:
        args.gemm = "ffma"                             # the pool / LSTM aggregators are built for fp32 only
    gemm = B.GEMM_BF16 if args.gemm == "bf16" else B.GEMM_FFMA
    agg_kw = {}
    if pool:
        from synth.graphs import pool_weights
        Wps, bps = pool_weights(cfg.dims)
        agg_kw = dict(aggregator=B.AGG_POOL, Wps=Wps, bps=bps)
    if lstm:
        from synth.graphs import lstm_weights
        agg_kw = dict(aggregator=B.AGG_LSTM, lstm=lstm_weights(cfg.dims))
    if gat:
        from synth.graphs import gat_weights
        Ws, bs, als, ars = gat_weights(cfg.dims)
        agg_kw = dict(aggregator=B.AGG_GAT, gat=(als, ars))
    feat_dtype = B.BF16 if args.gemm == "bf16" else B.FP32
    feats = X
    if not sharded and feat_dtype == B.BF16 and feats.dtype != torch.bfloat16:
        feats = feats.to(torch.bfloat16).contiguous()      # k/128 features are exact in bf16
    sim = args.world_sim if world == 1 and args.world_sim > 1 else 0
    plan_world = sim or world                     # #GPUs the plan is made for (R24 k_min, LPT ranks)
    kmin = max(cfg.k_min, plan_world)
    kmult = plan_world if args.rank_balanced_k else 1
    budget = cfg.mem_budget
    graph = DeviceGraph(rp, col)
    # C of Eq. 1 ("offline graph analysis"): exact, on the GPU, once per graph,
    # outside the timed region (buffalo_triangles + buffalo_avg_clustering, reading R27)
    t_c = time.perf_counter()
    _, C_eq1, C_ppm = B.clustering(graph.g)
    t_c = time.perf_counter() - t_c
    rep = AllgatherReplay(sim) if (sim and args.sim_shared) else None
    tr = Trainer(graph, feats, y, seeds, cfg.dims,
                 cfg.fanout, cfg.F, Ws, bs, feat_dtype=feat_dtype, gemm_mode=gemm, mem_budget=budget,
                 C_ppm=C_ppm, k_min=kmin, k_max=max(kmin, cfg.k_max), rank=rank, world=plan_world, process_group=pg,
                 pipeline=not args.no_pipeline, k_multiple=kmult, allgather=rep.fn if rep else None, **agg_kw)
    tr._sim_replay = rep
    full_batch_edges = None
    if args.config in ("products", "papers", "arxiv_lstm") + SHARDED:
        # calibrate M_ctr once so that one GPU needs >= 8 groups (products; 2 for the LSTM
        # workload), then freeze it for every N
        B_full = Trainer(graph, feats, y, seeds, cfg.dims,
                         cfg.fanout, cfg.F, Ws, bs, feat_dtype=feat_dtype, gemm_mode=gemm, C_ppm=C_ppm,
                         k_min=1, k_max=1, sample_cache=False, **agg_kw)
        _, _, est1, _ = B_full.schedule(0)
        full_batch_edges = int(B_full.sizes_h[0, cfg.L + 1:].sum())       # K = 1: no redundancy
        del B_full
        tr.sched.mem_budget = int(est1[0]) // (2 if args.config == "arxiv_lstm" else 8)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()

    if sim:
        return run_world_sim(args, tr, sim, flush, stream)
    prof_counters = torch.zeros(1 << 16, dtype=torch.int64, device="cuda")
    lr = 0.01
    for i in range(args.warmup):
        tr.run_epoch(epoch=i, lr=lr)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    clocks = Clocks(dev)
    clocks.start()
    # live roofline of the dominant kernel (k_gather_rows, the Aggregate): CUDA events around
    # each of its launches on its stream, algorithmic bytes from the edges it aggregated
    B.profile_begin("lstm_gates" if lstm else "pool_max" if pool else "gat_attn" if gat else "gather", prof_counters)
    l0 = B.launch_count()
    step_ms, edges, sizes, ks = [], 0, [], []
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    for i in range(args.steps):
        flush.zero_()                                  # L2 flushed between timed steps (outside events)
        s0 = torch.cuda.Event(enable_timing=True)
        s1 = torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        st = tr.run_epoch(epoch=args.warmup + i, lr=lr)
        s1.record(stream)
        s1.synchronize()
        step_ms.append(s0.elapsed_time(s1))
        edges += st["edges"]
        ks.append(st["K"])
        last_st = st
        sizes += [(g["n"], g["e"]) for g in st["groups"]]
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    launches = B.launch_count() - l0
    clk = clocks.stop()
    g_ms, g_launches, g_bytes = B.profile_end()
    total_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([total_ms, edges], dtype=torch.float64, device="cuda")
        mx = t.clone()
        torch.distributed.all_reduce(mx, op=torch.distributed.ReduceOp.MAX)
        sm = t.clone()
        torch.distributed.all_reduce(sm, op=torch.distributed.ReduceOp.SUM)
        total_ms, edges = float(mx[0]), float(sm[1])
    value = edges / (total_ms / 1e3)

    # end to end through the public API with host buffers: H2D of the step's seed batch from
    # pinned memory, D2H of the loss, copies inside the timed region
    seeds_h = seeds.cpu().pin_memory()
    loss_h = torch.empty(1, dtype=torch.float32).pin_memory()
    e2e_ms, e2e_edges = [], 0
    for i in range(max(1, args.steps)):
        flush.zero_()
        s0 = torch.cuda.Event(enable_timing=True)
        s1 = torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        if tr.pipeline:
            # the seed batch of step i+1 goes up (pinned H2D on the scheduler's stream) before the
            # plan made for it during step i; the plan used by step i was made for the batch sent
            # during step i-1 (the first e2e step schedules its batch itself: epoch mismatch)
            st = tr.run_epoch(epoch=1000 + i, lr=lr, next_seeds=seeds_h)
        else:
            tr.set_seeds(seeds_h)
            st = tr.run_epoch(epoch=1000 + i, lr=lr)
        loss_h.copy_(tr.loss, non_blocking=True)
        s1.record(stream)
        s1.synchronize()
        e2e_ms.append(s0.elapsed_time(s1))
        e2e_edges += st["edges"]
    e2e_val = e2e_edges / (sum(e2e_ms) / 1e3)
    if world > 1:
        t = torch.tensor([sum(e2e_ms), e2e_edges], dtype=torch.float64, device="cuda")
        mx = t.clone()
        torch.distributed.all_reduce(mx, op=torch.distributed.ReduceOp.MAX)
        sm = t.clone()
        torch.distributed.all_reduce(sm, op=torch.distributed.ReduceOp.SUM)
        e2e_val = float(sm[1]) / (float(mx[0]) / 1e3)

    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(peaks_path):
        peak, peak_src = json.load(open(peaks_path))["hbm_gbs"], "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    else:
        peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
    achieved = g_bytes / (g_ms / 1e3) / 1e9 if g_ms > 0 else 0.0
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        traffic = json.load(open(tpath)).get(f"{args.config}/{args.gemm}" + ("" if args.aggregator == "mean" else
                                                                              "/" + args.aggregator))
    # diagnostics outside the timed region: measured memory high-water of every own group of
    # the first timed epoch, and one sequential epoch's phase breakdown + block-build rates
    mem_est = measured_memory(tr, args.warmup)
    phases, build_rates = phase_breakdown(tr, args.warmup)
    if lstm:   # the LSTM path is bound by its gate GEMMs (fp32 as 3xTF32 on tcgen05): FLOP roofline
        tf = g_bytes / (g_ms / 1e3) / 1e12 if g_ms > 0 else 0.0
        if os.path.exists(peaks_path):
            bf = json.load(open(peaks_path))["bf16_tflops"]
            src = "measured bf16 (MEASURED_PEAKS.json bf16_tflops)"
        else:
            bf, src = 2250.0, "nominal bf16 (B200_PROFILING.md)"
        tpk = bf * (1.1 / 2.25) / 3.0      # tf32 = bf16 x the guide's 1.1 / 2.25 ratio; 3 TF32 products per fp32 one
        roof = {"bound": "tensor",
                "kernel": "k_tcf_gemm_tma (LSTM gate GEMMs of every step, fp32 as 3xTF32 on tcgen05 kind::tf32)",
                "achieved": tf, "peak": tpk, "unit": "TFLOP/s", "frac": tf / tpk, "traffic": None,
                "peak_source": src + " x 1.1/2.25 (tf32, B200_PROFILING.md nominal ratio) / 3 (hi*hi + hi*lo + "
                               "lo*hi TF32 products per fp32 product); achieved counts useful fp32 flops",
                "flops_per_launch": g_bytes / max(1, g_launches), "launch_ms": g_ms / max(1, g_launches),
                "launches": g_launches, "share_of_step": g_ms / total_ms}
    else:
        roof = {"bound": "hbm",
                "kernel": ("k_pool_max (GraphSAGE-pool neighbour max + argmax)" if pool else
                           "k_gat_attn (GAT edge softmax + attention-weighted neighbour sum)" if gat else
                           "k_gather_v2 (Aggregate: fwd neighbour mean, bwd transposed sum)" if gemm == B.GEMM_BF16
                           else "k_agg_rows / k_aggT (fp32 Aggregate of the FFMA parity path: fwd neighbour mean, "
                                "bwd transposed sum)"),
                "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "peak_source": peak_src,
                "algorithmic_bytes_per_launch": g_bytes / max(1, g_launches),
                "launch_ms": g_ms / max(1, g_launches), "launches": g_launches,
                "share_of_step": g_ms / total_ms}
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline and not (pool or lstm or gat or big):   # (the pool oracle is loop-plain: tests only)
            rp_h, col_h, X_h, y_h, seeds_h = host_copies(rp, col, X, y, tr.seeds)
            cpu = oracle_sample(cfg, rp_h, col_h, X_h, y_h, seeds_h, Ws, bs, args.cpu_baseline_seconds,
                                edges / args.steps)
        line = dict(
            metric="aggregated edges/s (epoch of Buffalo hot path)", value=value, unit="edges/s",
            n_gpus=world, steps=args.steps, warmup=args.warmup, ms_per_step=total_ms / args.steps,
            higher_is_better=True, scaling="strong", vs_baseline=None,
            dtype="bf16" if gemm == B.GEMM_BF16 else "f32", data="synthetic",
            config={"workload": WORKLOADS[args.config].replace(
                        "SAGE-mean", {"mean": "SAGE-mean", "pool": "SAGE-pool", "lstm": "SAGE-LSTM",
                                      "gat": "GAT (one head)"}[args.aggregator]),
                    "config": args.config, "K": ks[-1],
                    "gemm": args.gemm, "aggregator": args.aggregator,
                    "l2": "flushed (512 MiB write) between timed steps",
                    "epoch_ms": total_ms / args.steps, "edges_per_epoch": edges / args.steps,
                    "full_batch_edges": full_batch_edges,
                    "redundancy": (edges / args.steps / full_batch_edges) if full_batch_edges else None,
                    "phases_ms_sequential": phases, "block_build": build_rates,
                    "parallelism": f"dp{world} over bucket groups",
                    "feature_shards": ((8 if world == 1 else world) if sharded else None),
                    "pipeline": "scheduler of epoch e+1 overlapped with epoch e" if not args.no_pipeline else "off",
                    "C_eq1": C_eq1, "C_ppm": C_ppm, "C_table2": C_TABLE2.get(args.config),
                    "C_seconds": t_c},
            roofline=roof,
            cpu_baseline=cpu,
            e2e={"value": e2e_val, "unit": "edges/s", "h2d_bytes_per_step": 4 * len(seeds),
                 "d2h_bytes_per_step": 4},
            gpu_launches=launches, clocks=clk, memory=mem_est)
        print(json.dumps(line), flush=True)
    if shard_close is not None:
        torch.distributed.barrier()          # every rank is done reading the peers' shards
        shard_close()
    if world > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


def main():
    args = parse()
    cfg = CONFIGS[args.config]
    if args.impl == "reference":
        run_reference(args, cfg)
    else:
        run_ours(args, cfg)


if __name__ == "__main__":
    main()
