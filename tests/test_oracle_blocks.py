"""Pins for the oracle's sampling and block generation.

What pins them (not the oracle itself):
* Floyd sampling: size = min(deg, f), distinct, sorted, inside the row; chi-square uniformity
  over all C(deg, f) subsets (the defining property of sampling without replacement, R2).
* full-neighbour blocks are exactly the CSR slices (no sampling involved);
* blocks vs a brute-force set/dict construction (dst prefix, then ascending global id, R3/R4);
* invariants of the north star: block edges are a subset of the graph, dst is a prefix of
  src, src unique, n_{l-1} = |dst u N_s(dst)|; transposed block by its definition.
"""
import itertools

import numpy as np
import pytest
from scipy.stats import chi2

import oracle as O
from synth.graphs import random_graph, seed_nodes


def _graph(N=60, E=200, kind="powerlaw"):
    rp, col = random_graph(N, E, kind)
    return O.Graph(rp, col)


def test_sample_row_basic_properties():
    g = _graph(200, 1500)
    for v in range(g.N):
        deg = int(g.degree(v))
        row = g.col[g.row_ptr[v]:g.row_ptr[v + 1]]
        for f in (0, 1, 3, 10):
            s = O.sample_row(g, v, f, seed=7, hop=1)
            exp_n = deg if (f <= 0 or deg <= f) else f
            assert s.size == exp_n
            assert len(set(s.tolist())) == s.size                      # distinct
            assert set(s.tolist()) <= set(row.tolist())                # inside the row
            pos = np.searchsorted(row, s)
            assert np.all(np.diff(pos) > 0)                            # CSR (position) order
            if f <= 0 or deg <= f:
                assert np.array_equal(s, row)                          # all neighbours


def test_sample_row_uniform_over_subsets():
    # a star: node 0 has degree 6; every 3-subset of its 6 neighbours must be equally likely
    rp = np.array([0, 6, 7, 8, 9, 10, 11, 12], dtype=np.int64)
    col = np.array([1, 2, 3, 4, 5, 6, 0, 0, 0, 0, 0, 0], dtype=np.int32)
    g = O.Graph(rp, col)
    subsets = {c: 0 for c in itertools.combinations(range(1, 7), 3)}
    n = 40000
    for seed in range(n):
        subsets[tuple(O.sample_row(g, 0, 3, seed, 1).tolist())] += 1
    obs = np.array(list(subsets.values()), dtype=np.float64)
    exp = n / len(subsets)
    stat = float(((obs - exp) ** 2 / exp).sum())
    assert stat < chi2.ppf(1 - 1e-4, len(subsets) - 1), stat


def test_sample_depends_on_node_and_hop_only():
    g = _graph(300, 3000)
    v = int(np.argmax(np.diff(g.row_ptr)))
    a = O.sample_row(g, v, 5, 11, 1)
    assert np.array_equal(a, O.sample_row(g, v, 5, 11, 1))
    others = [O.sample_row(g, v, 5, 11, 2), O.sample_row(g, v, 5, 12, 1)]
    assert any(not np.array_equal(a, o) for o in others)


def _brute_blocks(g, seeds, L, fanout, seed):
    dst = [int(s) for s in seeds]
    out = [None] * L
    for l in range(L, 0, -1):
        rows = [O.sample_row(g, v, fanout[l - 1], seed, L - l + 1).tolist() for v in dst]
        src = list(dst) + sorted({u for r in rows for u in r} - set(dst))      # R3
        where = {v: i for i, v in enumerate(src)}
        out[l - 1] = dict(dst=list(dst), rows=rows, src=src, where=where)
        dst = src
    return out


@pytest.mark.parametrize("fanout", [[3, 4], [0, 0], [2, 0, 5]])
def test_blocks_vs_brute_force(fanout):
    g = _graph(80, 400)
    L = len(fanout)
    seeds = seed_nodes(g.N, 17)
    blocks = O.build_blocks(g, seeds, L, fanout, seed=3)
    ref = _brute_blocks(g, seeds, L, fanout, 3)
    edges = set(zip(np.repeat(np.arange(g.N), np.diff(g.row_ptr)).tolist(), g.col.tolist()))
    for l in range(1, L + 1):
        b, r = blocks[l - 1], ref[l - 1]
        assert b["n_dst"] == len(r["dst"]) and b["n_src"] == len(r["src"])
        assert b["src_global"].tolist() == r["src"]
        assert b["src_global"][: b["n_dst"]].tolist() == r["dst"]             # dst prefix
        assert len(set(r["src"])) == len(r["src"])                            # src unique
        flat = [u for row in r["rows"] for u in row]
        assert b["col_global"].tolist() == flat
        assert b["col_local"].tolist() == [r["where"][u] for u in flat]
        assert b["src_global"][b["col_local"]].tolist() == flat
        for i, row in enumerate(r["rows"]):
            for u in row:
                assert (r["dst"][i], u) in edges                             # edges subset
        assert b["n_src"] == len(set(r["dst"]) | set(flat))
        # every non-prefix src has at least one edge
        has_edge = np.zeros(b["n_src"], bool)
        has_edge[b["col_local"]] = True
        assert has_edge[b["n_dst"]:].all()
        # transposed block: for each src j, the dst i with an edge to j, ascending
        for j in range(b["n_src"]):
            exp = [i for i, row in enumerate(r["rows"]) if r["src"][j] in row]
            assert b["t_col"][b["t_row_ptr"][j]:b["t_row_ptr"][j + 1]].tolist() == exp


def test_full_neighbour_blocks_are_csr_slices():
    g = _graph(120, 700)
    seeds = seed_nodes(g.N, 30)
    blocks = O.build_blocks(g, seeds, 2, [0, 0], seed=1)
    for b in blocks:
        dst = b["src_global"][: b["n_dst"]]
        for i, v in enumerate(dst):
            row = g.col[g.row_ptr[v]:g.row_ptr[v + 1]]
            assert np.array_equal(b["col_global"][b["row_ptr"][i]:b["row_ptr"][i + 1]], row)


def test_group_blocks_subset_of_full_batch():
    g = _graph(150, 900)
    seeds = seed_nodes(g.N, 60)
    full = O.build_blocks(g, seeds, 2, [4, 6], seed=5)
    for part in np.array_split(seeds, 3):
        sub = O.build_blocks(g, part, 2, [4, 6], seed=5)
        for l in range(2):
            assert set(sub[l]["src_global"].tolist()) <= set(full[l]["src_global"].tolist())


def test_block_sizes_match_blocks():
    g = _graph(100, 500)
    seeds = seed_nodes(g.N, 25)
    n, e = O.block_sizes(g, seeds, 3, [2, 3, 4], 9)
    b = O.build_blocks(g, seeds, 3, [2, 3, 4], 9)
    assert n == [b[0]["n_src"], b[0]["n_dst"], b[1]["n_dst"], b[2]["n_dst"]]
    assert e == [b[0]["n_edges"], b[1]["n_edges"], b[2]["n_edges"]]
