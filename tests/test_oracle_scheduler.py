"""Pins for the oracle's scheduler: DegreeBucketing (Alg. 3 l.1), SplitExplosionBucket,
MemBalancedGrouping (Alg. 4), Eq. 1-2 and the memory model.

Pins: the paper's worked bucket example (tests/golden/fig7_buckets.txt),
the Range split example (tests/golden/range_split.txt), a hand-checked LPT
run, Graham's LPT bound (4/3 - 1/(3K)) against exhaustive optimum, the Fig. 9 grouping
structure on a constructed instance, hand values of Eq. 1, a hand-computed
memory-model instance, and plan invariants (every seed in exactly one group; estimates
within M_ctr; K minimal).
"""
import itertools
import math

import numpy as np
import pytest

import oracle as O
from conftest import read_golden
from synth.graphs import random_graph, seed_nodes


def _fig_graph():
    edges, buckets = [], {}
    for ln in read_golden("fig7_buckets.txt"):
        t = ln.split()
        if t[0] == "edge":
            edges.append((int(t[1]), int(t[2])))
        else:
            F = int(t[1].split("=")[1])
            d = int(t[2].rstrip(":"))
            buckets.setdefault(F, {})[d] = [int(x) for x in t[3:]]
    N = 12
    rows = [[] for _ in range(N)]
    for u, v in edges:
        rows[u].append(v)
        rows[v].append(u)
    rp = np.zeros(N + 1, np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    col = np.array([c for r in rows for c in sorted(r)], np.int32)
    return O.Graph(rp, col), buckets


@pytest.mark.parametrize("F", [4, 5, 7])
def test_degree_bucketing_paper_example(F):
    g, golden = _fig_graph()
    seeds = np.arange(12)
    D, bucket, order, hist = O.degree_bucketing(g, seeds, f_L=0, F=F)
    got = {}
    for p in order:
        got.setdefault(int(bucket[p]), []).append(int(seeds[p]))
    exp = golden[min(F, 5) if F <= 5 else 5]
    assert got == exp
    assert hist.sum() == 12


def test_degree_bucketing_fanout_caps_degree():
    g, _ = _fig_graph()
    D, bucket, _, _ = O.degree_bucketing(g, np.arange(12), f_L=3, F=10)
    assert D.max() == 3 and bucket.tolist() == np.minimum(g.degree(np.arange(12)), 3).tolist()


def test_split_is_range_partition():
    lines = read_golden("range_split.txt")
    inp = [int(x) for x in lines[0].split()[1:]]
    K = int(lines[1].split()[1])
    parts = [[int(x) for x in ln.split()[1:]] for ln in lines[2:]]
    assert [p.tolist() for p in O.split_explosion(inp, K)] == parts
    # uneven: the first (O mod K) pieces get one extra seed
    assert [len(p) for p in O.split_explosion(list(range(10)), 4)] == [3, 3, 2, 2]


def test_grouping_weight_eq1_hand_values():
    # R = min(1, I / (O*D*C)); O*D = E
    assert O.grouping_weight(1000, I=50, E=100, C_ppm=250_000) == 1000     # 50/(25) >= 1
    assert O.grouping_weight(1000, I=10, E=100, C_ppm=500_000) == 200      # 10/50 = 0.2
    assert O.grouping_weight(999, I=1, E=3, C_ppm=1_000_000) == 333        # floor(999/3)
    assert O.grouping_weight(1000, I=7, E=0, C_ppm=500_000) == 1000        # E = 0 => R = 1
    assert O.grouping_weight(1000, I=7, E=9, C_ppm=0) == 1000              # no C => R = 1


def _items(ws):
    return [dict(d=i, k=0, M=w, w=w) for i, w in enumerate(ws)]


def test_lpt_hand_example():
    ok, groups, loads = O.mem_balanced_grouping(_items([3, 7, 5, 6, 4]), 2, 14)
    assert ok and sorted(loads) == [11, 14]
    assert sorted(sorted(it["w"] for it in g) for g in groups) == [[3, 4, 7], [5, 6]]
    ok, _, _ = O.mem_balanced_grouping(_items([3, 7, 5, 6, 4]), 2, 13)
    assert not ok


def test_lpt_graham_bound_vs_exhaustive():
    rng = np.random.default_rng(1)
    for _ in range(60):
        n = int(rng.integers(3, 9))
        K = int(rng.integers(2, 4))
        ws = rng.integers(1, 100, n).tolist()
        _, _, loads = O.mem_balanced_grouping(_items(ws), K, 10**9)
        opt = min(max(sum(w for w, a in zip(ws, asg) if a == k) for k in range(K))
                  for asg in itertools.product(range(K), repeat=n))
        assert max(loads) <= (4 / 3 - 1 / (3 * K)) * opt + 1e-9


def test_fig9_grouping_structure():
    # group0 = degree-{2,3,4,5} + micro-bucket 0 of the split degree-10 bucket,
    # group1 = degree-{1,6,7,8,9} + micro-bucket 1 (weights constructed; the figure's are an image)
    w = {1: 31, 2: 42, 3: 25, 4: 51, 5: 14, 6: 7, 7: 32, 8: 2, 9: 58}
    items = [dict(d=d, k=0, M=v, w=v) for d, v in w.items()]
    items += [dict(d=10, k=0, M=114, w=114), dict(d=10, k=1, M=111, w=111)]
    ok, groups, _ = O.mem_balanced_grouping(items, 2, 10**9)
    key = lambda it: ("m", it["k"]) if it["d"] == 10 else it["d"]
    assert {key(i) for i in groups[0]} == {2, 3, 4, 5, ("m", 0)}
    assert {key(i) for i in groups[1]} == {1, 6, 7, 8, 9, ("m", 1)}


def test_mem_model_hand_instance():
    # L = 1, n = [5, 2], e = [3], dims = [4, 3]; every buffer rounds up to 256 B:
    # blocks: row_ptr, heavy, col_local, src_global, col_global = 5 * 256 = 1280
    # build frame: totals 256 + scan ws R(8*(ceil(257/4096)+2)) = 256 + partition counts
    #              R(4*(256+1)) = 1280  -> 1792
    # acts: agg R(2*8*4) + logits R(2*8*4) = 512
    # bwd frame l=1: dH_1 256 + dW partials R(1*3*8*4) 256 + db partials R(1*8*4) 256 = 768
    assert O.mem_model([5, 2], [3], [4, 3], O.FP32) == (1280 + 512 + 768, 1280 + 512 + 1792)
    # a wide layer: n = [40000, 20000], e = [100000], dims = [64, 32]
    # blocks: R(80004)=80128, R(80000)=80128, R(400000)=400128, R(160000)=160000, col_global 400128
    # build: 256 + R(8*(ceil(120001/4096)+2)) + counts R(4*(256*30+1)) = 256 + 256 + 30976
    # acts: agg R(20000*64*4)=5120000, logits R(20000*32*4)=2560000
    # bwd: dH R(20000*32*4)=2560000; splits: tiles=1*2 -> min(148, 40) = 40;
    #      dW R(40*32*128*4)=655360; db R(40*32*4)=5120
    blocks = 80128 + 80128 + 400128 + 160000 + 400128
    acts = 5120000 + 2560000
    bwd = 2560000 + 655360 + 5120
    assert O.mem_model([40000, 20000], [100000], [64, 32], O.FP32) == (blocks + acts + bwd,) * 2


def test_mem_model_monotone_and_bf16_smaller():
    a = O.mem_model([1000, 300, 50], [2000, 400], [64, 32, 8], O.FP32)
    b = O.mem_model([1000, 300, 60], [2000, 500], [64, 32, 8], O.FP32)
    assert b[0] >= a[0] and b[1] >= a[1]
    # bf16 activations halve the per-row terms; the bf16 backward's fixed db partial rows
    # (BWD_DB_PARTS x d) only matter for tiny micro-batches
    big = ([100000, 30000, 5000], [200000, 40000], [64, 32, 8])
    assert O.mem_model(*big, O.BF16)[0] < O.mem_model(*big, O.FP32)[0]


def _plan_invariants(plan, seeds, budget):
    gs = plan["group_seeds"]
    assert sorted(gs.tolist()) == sorted(seeds.tolist())                  # exactly once
    off = plan["group_offsets"]
    assert off[0] == 0 and off[-1] == seeds.size and np.all(np.diff(off) > 0)
    for k in range(plan["K"]):
        assert np.all(plan["group_of_seed"][np.isin(seeds, gs[off[k]:off[k + 1]])] == k)
    assert np.all(plan["est_bytes"] <= budget)


@pytest.mark.parametrize("fanout,F", [([3, 5], 5), ([0, 0], 6)])
def test_schedule_invariants_and_minimal_K(fanout, F):
    rp, col = random_graph(400, 3000, "powerlaw")
    g = O.Graph(rp, col)
    seeds = seed_nodes(g.N, 150)
    dims = [16, 32, 5]
    full = O.schedule(g, seeds, 2, fanout, F, 3, dims, k_min=1, k_max=1)
    assert full["K"] == 1
    budget = int(full["est_bytes"][0] * 0.45)
    plan = O.schedule(g, seeds, 2, fanout, F, 3, dims, mem_budget=budget)
    assert plan is not None and plan["K_tried"] >= 3
    _plan_invariants(plan, seeds, budget)
    # minimality: the same procedure with k_max = K - 1 fails
    assert O.schedule(g, seeds, 2, fanout, F, 3, dims, mem_budget=budget,
                      k_max=plan["K_tried"] - 1) is None
    # group seed order: items by (bucket asc, micro index asc), input order inside an item
    D, bucket, _, _ = O.degree_bucketing(g, seeds, fanout[-1], F)
    bpos = {int(s): int(bucket[i]) for i, s in enumerate(seeds)}
    off = plan["group_offsets"]
    for k in range(plan["K"]):
        bk = [bpos[int(s)] for s in plan["group_seeds"][off[k]:off[k + 1]]]
        assert bk == sorted(bk)


def test_schedule_budget_error_and_multi_gpu():
    rp, col = random_graph(200, 1200, "powerlaw")
    g = O.Graph(rp, col)
    seeds = seed_nodes(g.N, 80)
    assert O.schedule(g, seeds, 2, [3, 4], 4, 3, [8, 8, 3], mem_budget=1000, k_max=64) is None
    plan = O.schedule(g, seeds, 2, [3, 4], 4, 3, [8, 8, 3], num_gpus=4)
    assert plan["K"] == 4 and sorted(plan["rank_of_group"].tolist()) == [0, 1, 2, 3]


# ---------------------------------------------------------------- R7 / R25 pins
def _hand_stats(Ms, F):
    return {d: dict(M=M, w=M, O=10, I=1, E=1, pos=np.arange(1)) for d, M in Ms.items()}


def _pieces(M_F):
    def piece_stats(K):
        return [(k, dict(M=M_F // K + 10, w=M_F // K + 10, O=1, I=1, E=1, pos=np.arange(1))) for k in range(K)]
    return piece_stats


def test_explosion_flips_at_known_K():
    """Hand instance of R7 ("bucket explosion detected"): M_est = 200, 200 for
    the buckets of degree 1, 2 and 100 for bucket F = 3; sum M = 500, so M_F * K > 500 first
    holds at K = 6 (K = 5 is the equality, not an explosion).  At K = 6 the six micro-buckets
    (M = 100 // 6 + 10 = 26 each) are placed by Alg. 4: 200 -> g0, 200 -> g1, then pieces
    k0..k3 -> g2..g5, k4 -> g2 (lowest load, lowest index), k5 -> g3."""
    stats = _hand_stats({1: 200, 2: 200, 3: 100}, 3)
    for K, boom in ((2, False), (5, False), (6, True), (7, True)):
        res = O.core._alg3_k_loop(stats, 3, _pieces(100), 1000, 0, K, K)
        assert res is not None and res[0] == K and res[4] is boom, K
        assert len(res[1]) == (2 + K if boom else 3)
    K, items, groups, loads, boom = O.core._alg3_k_loop(stats, 3, _pieces(100), 1000, 0, 6, 6)
    got = [[(it["d"], it["k"]) for it in g] for g in groups]
    assert got == [[(1, 0)], [(2, 0)], [(3, 0), (3, 4)], [(3, 1), (3, 5)], [(3, 2)], [(3, 3)]]
    assert loads == [200, 200, 52, 52, 26, 26]
    # with a budget of 200 the loop succeeds at K = 3 without a split (the first feasible K)
    res = O.core._alg3_k_loop(stats, 3, _pieces(100), 200, 0, 1, 64)
    assert res[0] == 3 and res[4] is False
    # below 200 no K can succeed: the fast path stops at once, the plain loop tries every K
    calls = []

    def counting(K):
        calls.append(K)
        return _pieces(100)(K)
    assert O.core._alg3_k_loop(stats, 3, counting, 199, 0, 1, 64) is None and calls == []
    assert O.core._alg3_k_loop(stats, 3, counting, 199, 0, 1, 64, fast_paths=False) is None
    assert calls == list(range(6, 65))          # the plain loop splits at every exploding K


def test_fast_paths_equal_plain_loop_random():
    """R25: the scheduler's fast paths (skip a K when the never-split buckets cannot fit,
    stop when one of them alone exceeds M_ctr) give exactly the plan of the plain Alg. 3
    loop, on 200 random instances (graph shape, fanouts, F, budget, C, #GPUs)."""
    rng = np.random.default_rng(1234)
    graphs = [random_graph(n, p, kind) for n, p, kind in ((150, 600, "powerlaw"), (300, 2400, "powerlaw"),
                                                          (200, 500, "gnm"))]
    n_exploded = n_none = n_skipped = 0
    for it in range(200):
        rp, col = graphs[it % 3]
        g = O.Graph(rp, col)
        S = int(rng.integers(20, g.N))
        seeds = np.sort(rng.choice(g.N, S, replace=False)).astype(np.int32)
        L = int(rng.integers(1, 3))
        fan = [int(rng.choice([0, 2, 3, 5, 8])) for _ in range(L)]
        F = int(rng.integers(1, 9)) if fan[-1] <= 0 else min(fan[-1], int(rng.integers(1, 9)))
        dims = [int(rng.integers(4, 40)) for _ in range(L + 1)]
        full = O.schedule(g, seeds, L, fan, F, 3, dims, k_min=1, k_max=1)
        budget = int(full["est_bytes"][0] * rng.uniform(0.05, 1.1))
        kw = dict(mem_budget=budget, C_ppm=int(rng.choice([0, 0, 50000, 226000, 1000000])),
                  num_gpus=int(rng.choice([1, 1, 2, 3])), k_max=int(rng.integers(1, 13)))
        a = O.schedule(g, seeds, L, fan, F, 3, dims, **kw)
        b = O.schedule(g, seeds, L, fan, F, 3, dims, fast_paths=False, **kw)
        assert (a is None) == (b is None), it
        if a is None:
            n_none += 1
            continue
        n_exploded += bool(a["exploded"])
        n_skipped += a["K_tried"] > max(1, kw["num_gpus"])
        for k in ("K", "K_tried", "exploded", "num_items"):
            assert a[k] == b[k], (it, k)
        for k in ("group_offsets", "group_seeds", "group_of_seed", "est_bytes", "rank_of_group"):
            np.testing.assert_array_equal(a[k], b[k], err_msg=f"instance {it} {k}")
    # the instances exercise every branch
    assert n_exploded >= 10 and n_none >= 10 and n_skipped >= 10, (n_exploded, n_none, n_skipped)


def test_k_multiple_restricts_the_loop_to_multiples():
    """R31: with k_multiple = m the loop tries only multiples of m; the result is the first
    multiple at which the plain Alg. 3 step (run alone at that K) succeeds."""
    rng = np.random.default_rng(31)
    rp, col = random_graph(300, 2400, "powerlaw")
    g = O.Graph(rp, col)
    seen = 0
    for it in range(40):
        seeds = np.sort(rng.choice(g.N, int(rng.integers(40, 250)), replace=False)).astype(np.int32)
        fan, F, dims = [3, 5], 5, [16, 24, 5]
        full = O.schedule(g, seeds, 2, fan, F, 3, dims, k_min=1, k_max=1)
        budget = int(full["est_bytes"][0] * rng.uniform(0.08, 0.6))
        m = int(rng.choice([2, 3, 4]))
        a = O.schedule(g, seeds, 2, fan, F, 3, dims, mem_budget=budget, k_max=24, num_gpus=m, k_multiple=m)
        want = None
        for K in range(m, 25, m):
            if O.schedule(g, seeds, 2, fan, F, 3, dims, mem_budget=budget, k_min=K, k_max=K, num_gpus=m,
                          fast_paths=False) is not None:
                want = K
                break
        assert (a is None) == (want is None), it
        if a is not None:
            seen += 1
            assert a["K_tried"] == want and a["K_tried"] % m == 0
            assert sorted(a["group_seeds"].tolist()) == sorted(seeds.tolist())
    assert seen >= 20
