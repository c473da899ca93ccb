"""GPU parity of the triangle counting / average clustering coefficient C of Eq. 1
(reading R27) through the C ABI (buffalo_triangles,
buffalo_avg_clustering) against oracle.triangles / oracle.avg_clustering (plain C by
definition, pinned in tests/test_oracle_clustering.py).

T is an integer result: bit-exact on every node.  C is a float64 mean whose summation order
differs (oracle: node order; GPU: fixed tree), so |C_gpu - C_oracle| <= 1e-12 * max(C, 1e-300)
+ N * 2^-52 (rounding of N terms in [0, 1]); C_ppm equal unless C*10^6 sits within that bound of
a half-integer.  Inputs: synth/ only."""
import itertools
import math

import numpy as np
import pytest
import torch

import oracle as O
from synth.graphs import pairs_to_csr, random_graph

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from gpu_helpers import B


class _BareGraph:          # no node_map workspace: the clustering calls do not use it
    def __init__(self, rp, col):
        self.row_ptr = torch.as_tensor(rp).to("cuda", torch.int64).contiguous()
        self.col = torch.as_tensor(col).to("cuda", torch.int32).contiguous()
        self.g = B.Graph()
        self.g.num_nodes, self.g.nnz = self.row_ptr.numel() - 1, self.col.numel()
        self.g.row_ptr, self.g.col = self.row_ptr.data_ptr(), self.col.data_ptr()


def _gpu(rp, col):
    g = _BareGraph(rp, col)
    T, C, ppm = B.clustering(g.g)
    torch.cuda.synchronize()
    return g, T.cpu().numpy(), C, ppm


def _check_C(C, C_ref, ppm, N):
    tol = 1e-12 * abs(C_ref) + N * 2.0 ** -52
    assert abs(C - C_ref) <= tol, (C, C_ref)
    if abs(C_ref * 1e6 - math.floor(C_ref * 1e6) - 0.5) > 1e6 * tol:
        assert ppm == round(C_ref * 1e6)


def _graph(n, edges):
    pairs = np.array(sorted({(min(a, b), max(a, b)) for a, b in edges if a != b}), dtype=np.int64).reshape(-1, 2)
    return pairs_to_csr(n, pairs)


def test_closed_forms():
    rp, col = _graph(9, itertools.combinations(range(9), 2))     # K9: C = 1, T = C(8,2)
    _, T, C, ppm = _gpu(rp, col)
    assert np.all(T == 28) and C == 1.0 and ppm == 1_000_000
    n = 10                                                         # wheel W10
    rp, col = _graph(n + 1, [(0, i) for i in range(1, n + 1)] + [(i, i % n + 1) for i in range(1, n + 1)])
    _, T, C, _ = _gpu(rp, col)
    assert T[0] == n and np.all(T[1:] == 2)
    assert abs(C - (2.0 / (n - 1) + n * (2.0 / 3.0)) / (n + 1)) < 1e-15
    rp, col = _graph(8, [(0, i) for i in range(1, 6)])             # star + isolated nodes
    _, T, C, ppm = _gpu(rp, col)
    assert np.all(T == 0) and C == 0.0 and ppm == 0


def test_no_edges_and_single_node():
    for n in (1, 5):
        rp, col = np.zeros(n + 1, np.int64), np.zeros(0, np.int32)
        _, T, C, ppm = _gpu(rp, col)
        assert np.all(T == 0) and C == 0.0 and ppm == 0


@pytest.mark.parametrize("kind,N,E", [("gnm", 3000, 40000), ("powerlaw", 5000, 60000),
                                      ("powerlaw", 20000, 400000)])
def test_random_graphs_all_nodes(kind, N, E):
    rp, col = random_graph(N, E, kind)
    _, T, C, ppm = _gpu(rp, col)
    g = O.Graph(rp, col)
    T_ref = O.triangles(g)
    np.testing.assert_array_equal(T, T_ref)
    _check_C(C, O.avg_clustering(g, T_ref), ppm, N)


def test_deterministic_and_hub_rows():
    # a dense core (ranks tie on degree: the id breaks them) + long out(v) rows past the
    # shared-memory stage (a node adjacent to 3000 others of a clique-rich neighbourhood)
    rng = np.random.default_rng(7)
    n = 4000
    edges = [(0, i) for i in range(1, 3001)]
    edges += [tuple(x) for x in rng.integers(1, 3001, size=(60000, 2))]
    edges += list(itertools.combinations(range(3001, 3061), 2))
    rp, col = _graph(n, edges)
    g, T, C, _ = _gpu(rp, col)
    T2, C2, _ = B.clustering(g.g)
    assert np.array_equal(T2.cpu().numpy(), T) and C2 == C          # bit for bit, twice
    T_ref = O.triangles(O.Graph(rp, col))
    np.testing.assert_array_equal(T, T_ref)


def test_arxiv_shaped_full_graph():
    from synth import device as SD
    from synth.graphs import CONFIGS
    cfg = CONFIGS["arxiv"]
    rp, col = SD.random_graph(cfg.N, cfg.pairs, cfg.kind)
    g = _BareGraph(rp, col)
    T, C, ppm = B.clustering(g.g)
    rp_h, col_h = rp.cpu().numpy(), col.cpu().numpy()
    og = O.Graph(rp_h, col_h)
    T_ref = O.triangles(og)
    np.testing.assert_array_equal(T.cpu().numpy(), T_ref)
    _check_C(C, O.avg_clustering(og, T_ref), ppm, og.N)


def test_products_shaped_sampled_nodes():
    """At BASELINE.json configs[2]'s size: T of 3000 sampled nodes (degree <= 2000, the oracle
    tests every neighbour pair) bit for bit; invariants over all nodes (sum T divisible by 3,
    0 <= T_v <= d_v (d_v - 1) / 2, C in [0, 1])."""
    from synth import device as SD
    from synth.graphs import CONFIGS
    cfg = CONFIGS["products"]
    rp, col = SD.random_graph(cfg.N, cfg.pairs, cfg.kind)
    g = _BareGraph(rp, col)
    T, C, ppm = B.clustering(g.g)
    T = T.cpu().numpy()
    rp_h = rp.cpu().numpy()
    d = np.diff(rp_h)
    assert int(T.sum()) % 3 == 0 and np.all(T >= 0) and np.all(T <= d * (d - 1) // 2)
    assert 0.0 <= C <= 1.0 and ppm == round(C * 1e6)
    og = O.Graph(rp_h, col.cpu().numpy())
    rng = np.random.default_rng(11)
    cand = np.flatnonzero(d <= 2000)
    nodes = np.concatenate([rng.choice(cand, 2990, replace=False), cand[:10]])
    np.testing.assert_array_equal(T[nodes], O.triangles(og, nodes))
