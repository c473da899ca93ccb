"""synth.device (torch generator used by bench.py) is bit-identical to the numpy recipe."""
import numpy as np
import pytest
import torch

from synth import device as SD
from synth import graphs as G


def _check(dev, N, E, kind):
    rp, col = G.random_graph(N, E, kind)
    rp_d, col_d = SD.random_graph(N, E, kind, device=dev)
    assert np.array_equal(rp, rp_d.cpu().numpy())
    assert np.array_equal(col, col_d.cpu().numpy())
    x = G.features(N, 37, 48)
    assert np.array_equal(x, SD.features(N, 37, 48, device=dev).cpu().numpy())
    assert np.array_equal(G.labels(N, 13), SD.labels(N, 13, device=dev).cpu().numpy())
    assert np.array_equal(G.seed_nodes(N, N // 3), SD.seed_nodes(N, N // 3, device=dev).cpu().numpy())


@pytest.mark.parametrize("kind", ["powerlaw", "gnm"])
def test_device_generator_matches_numpy_cpu(kind):
    _check("cpu", 3000, 12000, kind)


def test_philox_words_match_numpy():
    from synth.philox import words
    c0 = np.arange(0, 5000, 7, dtype=np.uint64)
    a = words(0x123456789ABCDEF, c0, 3, 5, 1)
    b = SD.philox_words(0x123456789ABCDEF, torch.as_tensor(c0.astype(np.int64)), 3, 5, 1)
    for x, y in zip(a, b):
        assert np.array_equal(x.astype(np.int64), y.numpy())


@pytest.mark.gpu
@pytest.mark.parametrize("kind", ["powerlaw", "gnm"])
def test_device_generator_matches_numpy_gpu(kind):
    _check("cuda", 20000, 150000, kind)
