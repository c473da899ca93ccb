"""Philox4x32-10 pins: the synth (numpy) and oracle (C) generators against the Random123
known-answer vectors (tests/golden/philox_kat.txt).  The CUDA generator is pinned to the
same vectors in tests/test_gpu_parity.py."""
import numpy as np

from conftest import read_golden
from synth.philox import philox4x32_10
import oracle as O


def _kats():
    out = []
    for ln in read_golden("philox_kat.txt"):
        v = [int(x, 16) for x in ln.split()]
        out.append((v[0:4], v[4:6], v[6:10]))
    return out


def test_synth_philox_kat():
    for ctr, key, exp in _kats():
        got = philox4x32_10(*ctr, *key)
        assert [int(x) for x in got] == exp


def test_oracle_philox_kat():
    for ctr, key, exp in _kats():
        assert [int(x) for x in O.philox(ctr, key)] == exp


def test_synth_vs_oracle_stream():
    rng = np.random.default_rng(0)
    for _ in range(50):
        ctr = rng.integers(0, 2**32, 4, dtype=np.uint64)
        key = rng.integers(0, 2**32, 2, dtype=np.uint64)
        a = [int(x) for x in philox4x32_10(*ctr, *key)]
        b = [int(x) for x in O.philox(ctr.astype(np.uint32), key.astype(np.uint32))]
        assert a == b
