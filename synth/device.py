"""The same seeded inputs as `synth.graphs`, generated with torch tensor ops on a device.

Input infrastructure only (like the rest of `synth/`): graphs, features, labels and seeds,
bit-identical to the numpy recipe in `synth/graphs.py`, so that a bench run
on a products-shaped graph does not spend minutes generating it on one host core.  It holds
none of Buffalo's arithmetic.  `tests/test_gpu_parity.py::test_device_inputs_match_numpy`
checks bit-equality against the numpy generator.

Philox4x32-10 is evaluated on int64 tensors: the 32x32-bit products are split into 16-bit
halves so no intermediate leaves [0, 2^63) (no reliance on signed wrap-around).
"""
import math

import numpy as np
import torch

from .graphs import DATA_SEED, GRAPH_SEED, _CHUNK, _powerlaw_cdf
from .philox import TAG_FEAT, TAG_GRAPH, TAG_LABEL, TAG_MASK

_M0, _M1 = 0xD2511F53, 0xCD9E8D57
_W0, _W1 = 0x9E3779B9, 0xBB67AE85
_MASK = 0xFFFFFFFF


def _mulhilo(m, x):
    """(hi, lo) 32-bit words of the 64-bit product m * x, m a 32-bit constant, x int64 < 2^32."""
    xl = x & 0xFFFF
    xh = x >> 16
    pl = xl * m                       # < 2^48
    ph = xh * m                       # < 2^48
    mid = ph + (pl >> 16)             # < 2^49
    lo = ((mid & 0xFFFF) << 16) | (pl & 0xFFFF)
    hi = mid >> 16
    return hi & _MASK, lo & _MASK


def philox_words(seed, c0, c1, c2, c3):
    """Philox4x32-10 output words (int64 tensors holding uint32 values); counters broadcast."""
    seed = int(seed) & 0xFFFFFFFFFFFFFFFF
    ka, kb = seed & _MASK, seed >> 32
    t = [c if torch.is_tensor(c) else None for c in (c0, c1, c2, c3)]
    ref = next(x for x in t if x is not None)
    shape = torch.broadcast_shapes(*[x.shape for x in t if x is not None])
    xs = []
    for c in (c0, c1, c2, c3):
        if torch.is_tensor(c):
            xs.append((c.to(torch.int64) & _MASK).expand(shape))
        else:
            xs.append(torch.full(shape, int(c) & _MASK, dtype=torch.int64, device=ref.device))
    x0, x1, x2, x3 = xs
    for r in range(10):
        if r:
            ka = (ka + _W0) & _MASK
            kb = (kb + _W1) & _MASK
        hi0, lo0 = _mulhilo(_M0, x0)
        hi1, lo1 = _mulhilo(_M1, x2)
        x0, x1, x2, x3 = hi1 ^ x1 ^ ka, lo1, hi0 ^ x3 ^ kb, lo0
    return x0, x1, x2, x3


def _powerlaw_candidates(cdf, N, start, count, seed, dev):
    k = torch.arange(start, start + count, dtype=torch.int64, device=dev)
    w = philox_words(seed, k, 0, 0, TAG_GRAPH)
    scale = 1.0 / 9007199254740992.0
    ua = ((w[0] << 21) | (w[1] >> 11)).to(torch.float64) * scale
    ub = ((w[2] << 21) | (w[3] >> 11)).to(torch.float64) * scale
    u = torch.clamp(torch.searchsorted(cdf, ua, right=True), max=N - 1)
    v = torch.clamp(torch.searchsorted(cdf, ub, right=True), max=N - 1)
    return u, v


def _gnm_candidates(N, start, count, seed, dev):
    k = torch.arange(start, start + count, dtype=torch.int64, device=dev)
    w = philox_words(seed, k, 0, 0, TAG_GRAPH)
    # (w * N) >> 32 with w < 2^32, N < 2^31: split to stay below 2^63
    def scale(x):
        return ((x >> 16) * N + (((x & 0xFFFF) * N) >> 16)) >> 16
    return scale(w[0]), scale(w[1])


def undirected_keys(N, E, kind, seed=GRAPH_SEED, device="cuda"):
    """The E distinct undirected pairs (u < v) with the smallest first-draw index, as keys
    u * N + v (int64 [E], in first-draw order).  Memory-lean for billion-edge shapes: the
    candidates live in one growing buffer (draw order = position), a stable sort marks each
    key's first draw, and the E earliest first draws are cut by a prefix count."""
    dev = torch.device(device)
    cdf = torch.as_tensor(_powerlaw_cdf(N, 0.55, 10.0), device=dev) if kind == "powerlaw" else None
    target = int(E * 1.15) + 1024
    buf = torch.empty(target, dtype=torch.int64, device=dev)
    n = drawn = 0
    while True:
        while drawn < target:
            cnt = min(_CHUNK * 4, target - drawn)
            if kind == "powerlaw":
                u, v = _powerlaw_candidates(cdf, N, drawn, cnt, seed, dev)
            elif kind == "gnm":
                u, v = _gnm_candidates(N, drawn, cnt, seed, dev)
            else:
                raise ValueError(f"device generator: kind {kind!r} not supported")
            k = (torch.minimum(u, v) * N + torch.maximum(u, v))[u != v]
            del u, v
            if n + k.numel() > buf.numel():
                grown = torch.empty(max(n + k.numel(), int(buf.numel() * 1.5)), dtype=torch.int64, device=dev)
                grown[:n] = buf[:n]
                buf = grown
            buf[n:n + k.numel()] = k
            n += k.numel()
            drawn += cnt
        allk = buf[:n]
        sk, order = torch.sort(allk, stable=True)      # equal keys keep draw order: head = first draw
        head = torch.ones(n, dtype=torch.bool, device=dev)
        head[1:] = sk[1:] != sk[:-1]
        del sk
        fpos = order[head]
        del order, head
        if fpos.numel() >= E:
            first = torch.zeros(n, dtype=torch.bool, device=dev)
            first[fpos] = True
            del fpos
            c = torch.cumsum(first, 0, dtype=torch.int32 if n < (1 << 31) else torch.int64)
            cut = int(torch.searchsorted(c, torch.tensor([E], dtype=c.dtype, device=dev))[0])
            del c
            first[cut + 1:] = False                    # keep the E earliest first draws
            return allk[first]
        del fpos
        target = drawn + max(int((E - 0) * 0.2), _CHUNK)


def undirected_pairs(N, E, kind, seed=GRAPH_SEED, device="cuda"):
    """The E distinct undirected pairs (u < v) with the smallest first-draw index (int64 [E,2])."""
    sel = undirected_keys(N, E, kind, seed, device)
    return torch.stack([sel // N, sel % N], dim=1)


def pairs_to_csr(N, pairs):
    u, v = pairs[:, 0], pairs[:, 1]
    key = torch.sort(torch.cat([u * N + v, v * N + u]))[0]
    rows = key // N
    col = (key % N).to(torch.int32)
    counts = torch.bincount(rows, minlength=N)
    row_ptr = torch.zeros(N + 1, dtype=torch.int64, device=pairs.device)
    torch.cumsum(counts, 0, out=row_ptr[1:])
    return row_ptr, col


def keys_to_csr(N, sel, max_chunk=400_000_000):
    """Symmetric sorted CSR of the pairs sel = u * N + v (u < v), built in row ranges so that no
    more than ~max_chunk keys are sorted at once (the same CSR as pairs_to_csr)."""
    dev = sel.device
    lo = (sel // N).to(torch.int32)
    hi = (sel - lo.to(torch.int64) * N).to(torch.int32)
    deg = torch.bincount(lo, minlength=N) + torch.bincount(hi, minlength=N)
    row_ptr = torch.zeros(N + 1, dtype=torch.int64, device=dev)
    torch.cumsum(deg, 0, out=row_ptr[1:])
    del deg
    col = torch.empty(2 * sel.numel(), dtype=torch.int32, device=dev)
    nchunks = max(1, -(-2 * sel.numel() // max_chunk))
    bounds = [int(x) for x in torch.searchsorted(
        row_ptr, torch.linspace(0, 2 * sel.numel(), nchunks + 1, device=dev).to(torch.int64)).cpu()]
    bounds[0], bounds[-1] = 0, N
    for a, b in zip(bounds[:-1], bounds[1:]):
        if b <= a:
            continue
        m1 = (lo >= a) & (lo < b)
        m2 = (hi >= a) & (hi < b)
        key = torch.cat([lo[m1].to(torch.int64) * N + hi[m1], hi[m2].to(torch.int64) * N + lo[m2]])
        del m1, m2
        key = torch.sort(key)[0]
        col[int(row_ptr[a]):int(row_ptr[b])] = (key % N).to(torch.int32)
        del key
    return row_ptr, col


def random_graph(N, E, kind, seed=GRAPH_SEED, device="cuda"):
    return keys_to_csr(N, undirected_keys(N, E, kind, seed, device))


def features(N, d, pitch=None, seed=DATA_SEED, dtype=torch.float32, device="cuda"):
    """x[v][k] = ((w>>24)-128)/128 with w = word (k&3) of Philox(seed; v, 0, k>>2, tag 1)."""
    return features_range(0, N, d, pitch, seed, dtype, device)


def features_range(r0, r1, d, pitch=None, seed=DATA_SEED, dtype=torch.float32, device="cuda"):
    """Rows [r0, r1) of the feature table of `features` (one shard of a node-range sharded table)."""
    pitch = pitch or d
    out = torch.zeros((r1 - r0, pitch), dtype=dtype, device=device)
    nb = (d + 3) // 4
    rows = max(1, (_CHUNK * 4) // nb)
    blk = torch.arange(nb, dtype=torch.int64, device=device)[None, :]
    for s in range(r0, r1, rows):
        e = min(r1, s + rows)
        v = torch.arange(s, e, dtype=torch.int64, device=device)[:, None]
        w = philox_words(seed, v, 0, blk, TAG_FEAT)
        vals = torch.stack([(x >> 24) - 128 for x in w], dim=2).reshape(e - s, nb * 4)[:, :d]
        out[s - r0:e - r0, :d] = (vals.to(torch.float32) / 128.0).to(dtype)
    return out


def labels(N, classes, seed=DATA_SEED, device="cuda"):
    w = philox_words(seed, torch.arange(N, dtype=torch.int64, device=device), 0, 0, TAG_LABEL)[0]
    return (w % classes).to(torch.int32)


def seed_nodes(N, S, seed=DATA_SEED, device="cuda"):
    """The S nodes with the smallest (word0 of Philox(seed; v,0,0,tag 3), v), ascending."""
    if S >= N:
        return torch.arange(N, dtype=torch.int32, device=device)
    v = torch.arange(N, dtype=torch.int64, device=device)
    w = philox_words(seed, v, 0, 0, TAG_MASK)[0]
    key = (w << 31) | v                      # N < 2^31: same order as (w, v)
    sel = torch.topk(key, S, largest=False, sorted=False)[1]
    return torch.sort(sel)[0].to(torch.int32)
