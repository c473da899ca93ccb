"""Seeded synthetic inputs shaped like the paper's datasets (Table II, :375-382).

Input infrastructure only: graphs, features, labels, seeds and initial weights.  It
holds none of Buffalo's arithmetic (no sampling, bucketing, relabelling, grouping or
layer math) and is the ONE module that both the oracle tests and the CUDA-path tests /
bench draw their inputs from.

Recipe (restated in DESIGN.md):
* graphs are simple, symmetric, sorted CSR (row_ptr int64[N+1], col int32[2E]); power-law
  shapes use a Chung-Lu model: both endpoints of candidate k are drawn with probability
  proportional to (v + 10)^-0.55 from 53-bit uniforms of Philox(seed; k, 0, 0, tag 4)
  (node ids ascending = expected degree descending); self loops rejected; the graph is
  exactly the E distinct undirected pairs with the smallest first-draw index; Cora-sized
  uses uniform G(n, m) pairs with the same rule.  (R-MAT (0.57,0.19,0.19,0.05), the
  survey's first proposal, is kept as kind="rmat": at arxiv scale it leaves ~41% of the
  nodes isolated, far from Table II's average degree 13.7 — see DESIGN.md.)
* features x[v][k] = ((w >> 24) - 128) / 128, w = word (k&3) of Philox(seed; v, 0, k>>2,
  tag 1): values k/128, exact in fp32 and bf16;
* labels y_v = word0 of Philox(seed; v, 0, 0, tag 2) mod classes;
* seeds: the S nodes with the smallest (word0 of Philox(seed; v, 0, 0, tag 3), v), ascending id;
* weights: Xavier-uniform from Philox(seed; layer, row, col>>2, tag 5), biases 0 unless asked.
"""
import math
from dataclasses import dataclass, field

import numpy as np

from .philox import words, TAG_FEAT, TAG_LABEL, TAG_MASK, TAG_GRAPH, TAG_WEIGHT

GRAPH_SEED = 1
DATA_SEED = 2
SAMPLE_SEED = 3
WEIGHT_SEED = 5
INT64_MAX = (1 << 63) - 1

_CHUNK = 1 << 22


# ----------------------------------------------------------------------------- graphs
def _rmat_candidates(N, start, count, seed, a=0.57, b=0.19, c=0.19):
    """Candidate edges start..start+count-1 (u, v as int64), before rejection."""
    scale = max(1, math.ceil(math.log2(N)))
    t_a = int(round(a * 256))
    t_b = t_a + int(round(b * 256))
    t_c = t_b + int(round(c * 256))
    k = np.arange(start, start + count, dtype=np.uint64)
    u = np.zeros(count, dtype=np.int64)
    v = np.zeros(count, dtype=np.int64)
    n_calls = (scale + 15) // 16
    level = 0
    for j in range(n_calls):
        w = words(seed, k, j, 0, TAG_GRAPH)
        for wi in range(4):
            for byte in range(4):
                if level >= scale:
                    break
                q = ((w[wi] >> np.uint64(8 * byte)) & np.uint64(0xFF)).astype(np.int64)
                ubit = (q >= t_b).astype(np.int64)              # quadrants c, d
                vbit = (((q >= t_a) & (q < t_b)) | (q >= t_c)).astype(np.int64)  # b, d
                u = (u << 1) | ubit
                v = (v << 1) | vbit
                level += 1
    return u, v


def _powerlaw_cdf(N, alpha, v0):
    w = (np.arange(N, dtype=np.float64) + v0) ** (-alpha)
    cdf = np.cumsum(w)
    return cdf / cdf[-1]


_CDF_CACHE = {}


def _powerlaw_candidates(N, start, count, seed, alpha=0.55, v0=10.0):
    """Chung-Lu: both endpoints drawn with probability proportional to (v + v0)^-alpha."""
    key = (N, alpha, v0)
    if key not in _CDF_CACHE:
        _CDF_CACHE.clear()
        _CDF_CACHE[key] = _powerlaw_cdf(N, alpha, v0)
    cdf = _CDF_CACHE[key]
    k = np.arange(start, start + count, dtype=np.uint64)
    w = words(seed, k, 0, 0, TAG_GRAPH)
    scale = 1.0 / 9007199254740992.0   # 2^-53
    ua = ((w[0] << np.uint64(21)) | (w[1] >> np.uint64(11))).astype(np.float64) * scale
    ub = ((w[2] << np.uint64(21)) | (w[3] >> np.uint64(11))).astype(np.float64) * scale
    u = np.minimum(np.searchsorted(cdf, ua, side="right"), N - 1).astype(np.int64)
    v = np.minimum(np.searchsorted(cdf, ub, side="right"), N - 1).astype(np.int64)
    return u, v


def _gnm_candidates(N, start, count, seed):
    k = np.arange(start, start + count, dtype=np.uint64)
    w = words(seed, k, 0, 0, TAG_GRAPH)
    n = np.uint64(N)
    u = ((w[0] * n) >> np.uint64(32)).astype(np.int64)
    v = ((w[1] * n) >> np.uint64(32)).astype(np.int64)
    return u, v


def undirected_pairs(N, E, kind="rmat", seed=GRAPH_SEED):
    """The E distinct undirected pairs (u < v) with the smallest first-draw index."""
    gen = {"rmat": _rmat_candidates, "powerlaw": _powerlaw_candidates,
           "gnm": _gnm_candidates}[kind]
    keys, firsts = [], []
    drawn = 0
    target = int(E * 1.15) + 1024
    while True:
        while drawn < target:
            cnt = min(_CHUNK, target - drawn)
            u, v = gen(N, drawn, cnt, seed)
            ok = (u < N) & (v < N) & (u != v)
            lo = np.minimum(u, v)[ok]
            hi = np.maximum(u, v)[ok]
            keys.append(lo * N + hi)
            firsts.append(np.arange(drawn, drawn + cnt, dtype=np.int64)[ok])
            drawn += cnt
        allk = np.concatenate(keys)
        allf = np.concatenate(firsts)
        uk, idx = np.unique(allk, return_index=True)
        if uk.size >= E:
            order = np.argsort(allf[idx], kind="stable")[:E]
            sel = uk[order]
            return np.stack([sel // N, sel % N], axis=1)
        keys, firsts = [allk], [allf]
        target = drawn + max(int((E - uk.size) * 2.0), _CHUNK)


def pairs_to_csr(N, pairs):
    """Symmetrise undirected pairs into a sorted CSR (row_ptr int64[N+1], col int32)."""
    u = pairs[:, 0].astype(np.int64)
    v = pairs[:, 1].astype(np.int64)
    rows = np.concatenate([u, v])
    cols = np.concatenate([v, u])
    key = np.sort(rows * N + cols)
    rows = key // N
    col = (key % N).astype(np.int32)
    counts = np.bincount(rows, minlength=N).astype(np.int64)
    row_ptr = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return row_ptr, col


def random_graph(N, E, kind="rmat", seed=GRAPH_SEED):
    return pairs_to_csr(N, undirected_pairs(N, E, kind, seed))


# ----------------------------------------------------------------------------- node data
def features(N, d, pitch=None, seed=DATA_SEED, dtype=np.float32):
    """x[v][k] = ((w>>24)-128)/128; rows padded with zeros to `pitch` columns."""
    pitch = pitch or d
    out = np.zeros((N, pitch), dtype=dtype)
    nb = (d + 3) // 4
    for s in range(0, N, _CHUNK // max(1, nb)):
        e = min(N, s + _CHUNK // max(1, nb))
        v = np.arange(s, e, dtype=np.uint64)[:, None]
        blk = np.arange(nb, dtype=np.uint64)[None, :]
        w = words(seed, v, 0, blk, TAG_FEAT)
        vals = np.stack([((x >> np.uint64(24)).astype(np.int64) - 128) for x in w], axis=2)
        vals = vals.reshape(e - s, nb * 4)[:, :d].astype(np.float32) / np.float32(128.0)
        out[s:e, :d] = vals.astype(dtype)
    return out


def labels(N, classes, seed=DATA_SEED):
    w = words(seed, np.arange(N, dtype=np.uint64), 0, 0, TAG_LABEL)[0]
    return (w % np.uint64(classes)).astype(np.int32)


def seed_nodes(N, S, seed=DATA_SEED):
    """The S nodes with the smallest (word0 of Philox(seed; v,0,0,tag 3), v), ascending."""
    if S >= N:
        return np.arange(N, dtype=np.int32)
    w = words(seed, np.arange(N, dtype=np.uint64), 0, 0, TAG_MASK)[0]
    key = (w << np.uint64(32)) | np.arange(N, dtype=np.uint64)
    sel = np.argpartition(key, S - 1)[:S]
    return np.sort(sel).astype(np.int32)


def xavier_weights(dims, seed=WEIGHT_SEED, bias_scale=0.0):
    """Per layer l = 1..L: W_l float32 [d_l, 2*d_{l-1}] (Xavier-uniform) and b_l [d_l]."""
    Ws, bs = [], []
    for l in range(1, len(dims)):
        rows, cols = dims[l], 2 * dims[l - 1]
        a = math.sqrt(6.0 / (rows + cols))
        r = np.arange(rows, dtype=np.uint64)[:, None]
        c = np.arange(cols, dtype=np.uint64)[None, :]
        w = words(seed, l, r, c >> np.uint64(2), TAG_WEIGHT)
        sel = np.choose((c & np.uint64(3)).astype(np.int64), w)
        u = (sel.astype(np.float64) + 0.5) / 4294967296.0
        Ws.append(((2.0 * u - 1.0) * a).astype(np.float32))
        if bias_scale:
            wb = words(seed, l, rows + 7, np.arange(rows, dtype=np.uint64), TAG_WEIGHT)[0]
            ub = (wb.astype(np.float64) + 0.5) / 4294967296.0
            bs.append(((2.0 * ub - 1.0) * bias_scale).astype(np.float32))
        else:
            bs.append(np.zeros(rows, dtype=np.float32))
    return Ws, bs


def pool_weights(dims, seed=WEIGHT_SEED, bias_scale=0.0, dyadic=False):
    """GraphSAGE-pool weights per layer l = 1..L: W_pool_l float32 [d_{l-1}, d_{l-1}]
    (Xavier-uniform, Philox counter c0 = 64 + l so the stream is disjoint from the layer
    weights) and b_pool_l [d_{l-1}].  dyadic=True rounds every value to a multiple of 2^-8
    (exact products with k/128 features: the pool transform is then exact in fp32 for
    d_{l-1} <= 256, so float-decided argmaxes agree with the oracle)."""
    Wps, bps = [], []
    for l in range(1, len(dims)):
        d = dims[l - 1]
        a = math.sqrt(6.0 / (2 * d))
        r = np.arange(d, dtype=np.uint64)[:, None]
        c = np.arange(d, dtype=np.uint64)[None, :]
        w = words(seed, 64 + l, r, c >> np.uint64(2), TAG_WEIGHT)
        sel = np.choose((c & np.uint64(3)).astype(np.int64), w)
        u = (sel.astype(np.float64) + 0.5) / 4294967296.0
        W = (2.0 * u - 1.0) * a
        if bias_scale:
            wb = words(seed, 64 + l, d + 7, np.arange(d, dtype=np.uint64), TAG_WEIGHT)[0]
            b = ((wb.astype(np.float64) + 0.5) / 4294967296.0 * 2.0 - 1.0) * bias_scale
        else:
            b = np.zeros(d)
        if dyadic:
            W, b = np.round(W * 256.0) / 256.0, np.round(b * 256.0) / 256.0
        Wps.append(W.astype(np.float32))
        bps.append(b.astype(np.float32))
    return Wps, bps


def lstm_weights(dims, seed=WEIGHT_SEED):
    """GraphSAGE-LSTM weights per layer l = 1..L (hidden size d = d_{l-1}): W_ih, W_hh float32
    [4d, d] and b [4d] (b_ih + b_hh of nn.LSTM), uniform on +-1/sqrt(d) as nn.LSTM initialises
    them; Philox counters c0 = 128 + l (W_ih), 160 + l (W_hh), 192 + l (b)."""
    Wih, Whh, bl = [], [], []
    for l in range(1, len(dims)):
        d = dims[l - 1]
        a = 1.0 / math.sqrt(d)
        r = np.arange(4 * d, dtype=np.uint64)[:, None]
        c = np.arange(d, dtype=np.uint64)[None, :]
        out = []
        for c0 in (128 + l, 160 + l):
            w = words(seed, c0, r, c >> np.uint64(2), TAG_WEIGHT)
            sel = np.choose((c & np.uint64(3)).astype(np.int64), w)
            u = (sel.astype(np.float64) + 0.5) / 4294967296.0
            out.append(((2.0 * u - 1.0) * a).astype(np.float32))
        wb = words(seed, 192 + l, 0, np.arange(4 * d, dtype=np.uint64), TAG_WEIGHT)[0]
        ub = (wb.astype(np.float64) + 0.5) / 4294967296.0
        Wih.append(out[0])
        Whh.append(out[1])
        bl.append(((2.0 * ub - 1.0) * a).astype(np.float32))
    return Wih, Whh, bl


def gat_weights(dims, seed=WEIGHT_SEED, bias_scale=0.0):
    """GAT weights per layer l = 1..L (one head): W_l float32 [d_l, d_{l-1}] (Xavier-uniform),
    attention vectors a_l, a_r [d_l] (Xavier-uniform of a [2 d_l] vector as GATConv) and b_l
    [d_l]; Philox counters c0 = 224 + l (W), 240 + l (a), 248 + l (b)."""
    Ws, als, ars, bs = [], [], [], []
    for l in range(1, len(dims)):
        din, dout = dims[l - 1], dims[l]
        a = math.sqrt(6.0 / (din + dout))
        r = np.arange(dout, dtype=np.uint64)[:, None]
        c = np.arange(din, dtype=np.uint64)[None, :]
        w = words(seed, 224 + l, r, c >> np.uint64(2), TAG_WEIGHT)
        sel = np.choose((c & np.uint64(3)).astype(np.int64), w)
        u = (sel.astype(np.float64) + 0.5) / 4294967296.0
        Ws.append(((2.0 * u - 1.0) * a).astype(np.float32))
        aa = math.sqrt(6.0 / (1 + 2 * dout))
        wa = words(seed, 240 + l, 0, np.arange(2 * dout, dtype=np.uint64), TAG_WEIGHT)[0]
        ua = ((wa.astype(np.float64) + 0.5) / 4294967296.0 * 2.0 - 1.0) * aa
        als.append(ua[:dout].astype(np.float32))
        ars.append(ua[dout:].astype(np.float32))
        if bias_scale:
            wb = words(seed, 248 + l, 0, np.arange(dout, dtype=np.uint64), TAG_WEIGHT)[0]
            bs.append((((wb.astype(np.float64) + 0.5) / 4294967296.0 * 2.0 - 1.0) * bias_scale).astype(np.float32))
        else:
            bs.append(np.zeros(dout, dtype=np.float32))
    return Ws, bs, als, ars


# ----------------------------------------------------------------------------- configs
@dataclass
class Config:
    name: str
    N: int
    pairs: int
    kind: str
    d0: int
    classes: int
    hidden: int
    L: int
    fanout: list          # fanout[l-1] for block l (DGL order: input layer first); <=0 = all
    F: int                # cut-off degree
    S: int                # number of seeds (batch)
    k_min: int = 1
    k_max: int = 4096
    mem_budget: int = INT64_MAX
    C_ppm: int = 0        # 0 => measured on the generated graph (oracle tests) / R = 1
    extra: dict = field(default_factory=dict)

    @property
    def dims(self):
        return [self.d0] + [self.hidden] * (self.L - 1) + [self.classes]


CONFIGS = {
    # BASELINE.json configs[0]: Cora-sized, 2-layer SAGE-mean, fanout (10,25), 4 partitions.
    "cora": Config("cora", 2708, 5278, "gnm", 1433, 7, 256, 2, [10, 25], 25, 2708, 4, 4),
    # configs[1]: ogbn-arxiv-shaped, 3-layer, full-neighbour blocks (F = 10).
    "arxiv": Config("arxiv", 169343, 1166243, "powerlaw", 128, 40, 256, 3, [0, 0, 0], 10, 90941, 4, 4),
    # configs[2]: ogbn-products-shaped, 3-layer, fanout (10,25,30), budget forcing K >= 8.
    "products": Config("products", 2449029, 61859140, "powerlaw", 100, 47, 256, 3, [10, 25, 30], 30,
                       196615, 8, 4096),
    # The paper's LSTM workload: arxiv-shaped, 2-layer SAGE-LSTM, LSTM hidden 128,
    # cut-offs 25 (1-hop) and 10 (2-hop) = fanout (10, 25) in DGL order; budget forcing K >= 2.
    "arxiv_lstm": Config("arxiv_lstm", 169343, 1166243, "powerlaw", 128, 40, 128, 2, [10, 25], 25, 90941, 2,
                         4096),
    # configs[3]: ogbn-papers100M-shaped, 2-layer, fanout (10,25).
    "papers": Config("papers", 111059956, 1615685872, "powerlaw", 128, 172, 256, 2, [10, 25], 25,
                     1207179, 8, 4096),
    # configs[4]: IGB-large-shaped, 3-layer, fanout (5,10,15).
    "igb": Config("igb", 100000000, 1200000000, "powerlaw", 1024, 19, 256, 3, [5, 10, 15], 15,
                  1000000, 8, 4096),
    # configs[4] at 1/8 of the nodes, edges and seeds (one GPU's share of the 8-GPU run: a 25.6 GB
    # 1024-d bf16 table, held as 8 node-range shards), for the single-GPU bench and tests.
    "igb_small": Config("igb_small", 12500000, 150000000, "powerlaw", 1024, 19, 256, 3, [5, 10, 15], 15,
                        125000, 8, 4096),
}


def scaled(cfg, factor, name=None):
    """A smaller graph with the same shape (for parity tests that must finish in seconds)."""
    N = max(64, int(cfg.N * factor))
    pairs = max(N, int(cfg.pairs * factor))
    S = max(16, int(cfg.S * factor))
    return Config(name or f"{cfg.name}@{factor}", N, pairs, cfg.kind, cfg.d0, cfg.classes,
                  cfg.hidden, cfg.L, list(cfg.fanout), cfg.F, S, cfg.k_min, cfg.k_max,
                  cfg.mem_budget, cfg.C_ppm)


def make_inputs(cfg, feat_dtype=np.float32, pitch=None):
    row_ptr, col = random_graph(cfg.N, cfg.pairs, cfg.kind)
    x = features(cfg.N, cfg.d0, pitch or cfg.d0, dtype=feat_dtype)
    y = labels(cfg.N, cfg.classes)
    s = seed_nodes(cfg.N, cfg.S)
    return row_ptr, col, x, y, s
