"""Philox4x32-10 counter-based generator, vectorised over numpy arrays.

Input infrastructure only (shared by the CUDA path's tests/bench and the oracle's
tests): it holds none of Buffalo's arithmetic.  The same generator is implemented
independently in `oracle/buffalo_oracle.c` (oracle side) and in
`paper_conf_hpca_yangzl25_b200/csrc/philox.cuh` (CUDA side); all three are pinned to
the Random123 known-answer vectors in `tests/test_philox.py`.

Stream layout: key = (lo32(seed),
hi32(seed)); counter = (c0 = node/candidate id, c1 = hop or sub-stream, c2 = block
index j>>2, c3 = tag); draw j is word (j & 3).
Tags: 0 sampling, 1 features, 2 labels, 3 train mask, 4 graph generation, 5 weights.
"""
import numpy as np

M0 = np.uint64(0xD2511F53)
M1 = np.uint64(0xCD9E8D57)
W0 = np.uint64(0x9E3779B9)
W1 = np.uint64(0xBB67AE85)
MASK = np.uint64(0xFFFFFFFF)
S32 = np.uint64(32)

TAG_SAMPLE, TAG_FEAT, TAG_LABEL, TAG_MASK, TAG_GRAPH, TAG_WEIGHT = 0, 1, 2, 3, 4, 5


def _u64(x, shape=None):
    a = np.asarray(x, dtype=np.uint64) & MASK
    if shape is not None:
        a = np.broadcast_to(a, shape)
    return a


def philox4x32_10(c0, c1, c2, c3, k0, k1):
    """Return the four 32-bit output words (as uint64 arrays holding uint32 values)."""
    shape = np.broadcast_shapes(np.shape(c0), np.shape(c1), np.shape(c2), np.shape(c3))
    x0, x1, x2, x3 = (_u64(c, shape).copy() for c in (c0, c1, c2, c3))
    ka = _u64(k0, shape).copy()
    kb = _u64(k1, shape).copy()
    for r in range(10):
        if r:
            ka = (ka + W0) & MASK
            kb = (kb + W1) & MASK
        p0 = M0 * x0          # < 2^64: exact in uint64
        p1 = M1 * x2
        hi0, lo0 = p0 >> S32, p0 & MASK
        hi1, lo1 = p1 >> S32, p1 & MASK
        x0, x1, x2, x3 = hi1 ^ x1 ^ ka, lo1, hi0 ^ x3 ^ kb, lo0
    return x0, x1, x2, x3


def split_seed(seed):
    seed = int(seed) & 0xFFFFFFFFFFFFFFFF
    return seed & 0xFFFFFFFF, seed >> 32


def words(seed, c0, c1, c2, c3):
    k0, k1 = split_seed(seed)
    return philox4x32_10(c0, c1, c2, c3, k0, k1)
