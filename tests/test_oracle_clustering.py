"""Pins of the oracle's clustering coefficient (C of Eq. 1; reading R27):
closed forms on graphs whose triangles are known, and an independent brute force over node
triples on small random graphs."""
import itertools
import math

import numpy as np
import pytest

import oracle as O
from synth.graphs import pairs_to_csr, random_graph


def _graph(n, edges):
    pairs = np.array(sorted({(min(a, b), max(a, b)) for a, b in edges if a != b}), dtype=np.int64).reshape(-1, 2)
    rp, col = pairs_to_csr(n, pairs)
    return O.Graph(rp, col)


def test_complete_graph():
    n = 9
    g = _graph(n, itertools.combinations(range(n), 2))
    assert np.all(O.triangles(g) == math.comb(n - 1, 2))
    assert O.avg_clustering(g) == 1.0


@pytest.mark.parametrize("n", [3, 4, 7])
def test_cycle(n):
    g = _graph(n, [(i, (i + 1) % n) for i in range(n)])
    T = O.triangles(g)
    assert np.all(T == (1 if n == 3 else 0))
    assert O.avg_clustering(g) == (1.0 if n == 3 else 0.0)


def test_star_and_isolated_nodes():
    g = _graph(8, [(0, i) for i in range(1, 6)])          # nodes 6, 7 isolated
    assert np.all(O.triangles(g) == 0)
    assert O.avg_clustering(g) == 0.0


def test_wheel():
    n = 10                                                 # hub 0, rim 1..n
    edges = [(0, i) for i in range(1, n + 1)] + [(i, i % n + 1) for i in range(1, n + 1)]
    g = _graph(n + 1, edges)
    T = O.triangles(g)
    assert T[0] == n and np.all(T[1:] == 2)
    want = (2.0 / (n - 1) + n * (2.0 / 3.0)) / (n + 1)
    assert abs(O.avg_clustering(g) - want) < 1e-15


@pytest.mark.parametrize("kind", ["gnm", "powerlaw"])
def test_brute_force_triples(kind):
    rp, col = random_graph(60, 400, kind)
    g = O.Graph(rp, col)
    adj = [set(col[rp[v]:rp[v + 1]].tolist()) for v in range(60)]
    T = np.zeros(60, np.int64)
    for a, b, c in itertools.combinations(range(60), 3):
        if b in adj[a] and c in adj[a] and c in adj[b]:
            T[[a, b, c]] += 1
    np.testing.assert_array_equal(O.triangles(g), T)
    d = np.diff(rp)
    loc = [2 * T[v] / (d[v] * (d[v] - 1)) if d[v] >= 2 else 0.0 for v in range(60)]
    assert abs(O.avg_clustering(g) - sum(loc) / 60) < 1e-14
    # subset form = full form
    nodes = np.array([0, 5, 17, 59])
    np.testing.assert_array_equal(O.triangles(g, nodes), T[nodes])
