"""Pins of the oracle against what PAPER.md and the mathematics fix (CPU only).

P1 Fig. 1 trace, P2 Fig. 4(c) trace, P4 brute-force exactness, P5 greedy
special case, P9 Table III closed form, R7 distance closed forms, recall
definition.  Equivalence (P3), invariants (P6) and Bloom (P7) live in
test_oracle_equiv.py / test_oracle_bloom.py.
"""
import math

import numpy as np
import pytest

import oracle
from _golden import golden_path


def load_toy():
    rows, coords, states, result = {}, {}, {"fig1": {}, "fig4c": {}}, None
    with open(golden_path("fig1_fig4c_toy.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            if line.startswith("graph"):
                head, tail = line[len("graph"):].split(":")
                rows[int(head)] = [int(x) for x in tail.split()]
            elif line.startswith("coord"):
                _, v, c = line.split()
                coords[int(v)] = float(c)
            elif line.startswith("fig"):
                head, q, t, vis = [s.strip() for s in line.split("|")]
                fig, it = head.split()
                parse = lambda s: [] if s == "-" else [int(x) for x in s.split()]
                states[fig][int(it)] = (parse(q), parse(t), parse(vis))
            elif line.startswith("result"):
                result = [int(x) for x in line.split()[1:]]
    n = len(rows)
    adj = np.full((n, 4), -1, np.int32)
    for v, r in rows.items():
        adj[v - 1] = [x - 1 if x > 0 else -1 for x in r]
    data = np.array([[coords[v]] for v in range(1, n + 1)], np.float32)
    return data, adj, states, result


def run_traced(flags, L=3, K=3):
    data, adj, _, _ = load_toy()
    seen = {}

    def cb(it, q, t, vis):
        seen[it] = ([x + 1 for x in q], [x + 1 for x in t],
                    None if vis is None else [x + 1 for x in vis])

    ids, dists, ctr, capped = oracle.search(data, adj, np.zeros((1, 1), np.float32), K, L,
                                            flags=flags, trace=cb)
    assert capped == 0
    return seen, [int(x) + 1 for x in ids[0]], dists[0], ctr[0]


def test_fig1_trace_plain_algorithm1():
    """P1: Algorithm 1 literally (unbounded q, exact visited) reproduces every
    q / topk / visited state of Fig. 1 and the path's result."""
    _, _, states, result = load_toy()
    seen, ids, _, ctr = run_traced(oracle.PLAIN)
    for it, (q, t, vis) in states["fig1"].items():
        sq, st, sv = seen[it]
        assert sq == q, f"iteration {it}: q"
        assert sorted(st) == sorted(t), f"iteration {it}: topk"
        assert sv == sorted(vis), f"iteration {it}: visited"
    assert max(seen) == 4  # iteration 5 pops 3, worse than topk max 7 -> break
    assert ids == result
    # plain mode computes each visited vertex's distance exactly once: 10
    assert ctr[0] == len(states["fig1"][4][2]) == 10


def test_fig4c_trace_bounded_sel_del():
    """P2: bounded q (§IV-C) + selected insertion (§IV-D) + visited deletion
    (§IV-E) reproduce Fig. 4(c)'s states."""
    _, _, states, result = load_toy()
    seen, ids, _, ctr = run_traced(oracle.OPTIMIZED)
    for it, (q, t, vis) in states["fig4c"].items():
        sq, st, sv = seen[it]
        assert sq == q, f"iteration {it}: q"
        assert sorted(st) == sorted(t), f"iteration {it}: topk"
        assert sv == sorted(vis), f"iteration {it}: visited"
    assert ids == result
    # "we may compute its distance again": 4 and 1 are recomputed, so
    # 12 distance computations against plain mode's 10 (derived).
    assert ctr[0] == 12 and ctr[1] == 4
    # visited never exceeds |q| + |topk| <= 2K
    assert all(len(v) <= 6 for _, _, v in seen.values())


@pytest.mark.parametrize("flags", [oracle.PLAIN, oracle.BOUNDED_Q,
                                   oracle.BOUNDED_Q | oracle.SEL, oracle.OPTIMIZED,
                                   oracle.OPTIMIZED_BLOOM])
def test_toy_result_same_for_every_optimization(flags):
    """Observation 1 and P:431/P:435: the optimizations do not change
    the output; Fig. 4's panels all end at topk = {7, 2, 8}."""
    _, _, _, result = load_toy()
    _, ids, _, _ = run_traced(flags)
    assert ids == result


def test_table3_index_sizes_are_32_slots_per_vertex():
    """P9 / reading A8: Table III = ceil(n * 32 * 4 B / 2^20)."""
    with open(golden_path("table3_index_sizes.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            name, n, mb = line.split()
            assert math.ceil(int(n) * 32 * 4 / 2 ** 20) == int(mb), name
            # the paper's own "16" would give half; that is HNSW's M
            assert math.ceil(int(n) * 16 * 4 / 2 ** 20) != int(mb), name


def test_distance_closed_forms():
    """R7 / §VI: squared L2, negative inner product, 1 - cosine."""
    p = np.array([3.0, 4.0, 0.0, 0.0], np.float32)
    z = np.zeros(4, np.float32)
    assert oracle.distance(p, z, oracle.L2) == 25.0
    assert oracle.distance(p, np.array([3, 4, 0, 1], np.float32), oracle.L2) == 1.0
    assert oracle.distance(p, np.array([1, 1, 0, 0], np.float32), oracle.IP) == -7.0
    # cosine: parallel 0, orthogonal 1, antiparallel 2, zero norm 1
    assert oracle.distance(p, 2 * p, oracle.COSINE) == pytest.approx(0.0, abs=1e-7)
    assert oracle.distance(p, np.array([-4, 3, 0, 0], np.float32), oracle.COSINE) == 1.0
    assert oracle.distance(p, -p, oracle.COSINE) == 2.0
    assert oracle.distance(p, z, oracle.COSINE) == 1.0
    # -0.0 is canonicalised: IP of orthogonal vectors is +0.0
    d = oracle.distance(p, np.array([-4, 3, 0, 0], np.float32), oracle.IP)
    assert d == 0.0 and math.copysign(1.0, d) == 1.0
    # accumulation is fp64: catastrophic fp32 cancellation does not occur
    a = np.array([1e8, 1.0, -1e8], np.float32)
    b = np.array([1.0, 1.0, 1.0], np.float32)
    assert oracle.distance(a, b, oracle.IP) == -1.0


def numpy_topk(data, q, K, metric):
    """Independent brute force: fp64 distances, lexsort by (dist32, id)."""
    d64 = data.astype(np.float64)
    q64 = q.astype(np.float64)
    if metric == oracle.L2:
        d = ((d64 - q64) ** 2).sum(1)
    elif metric == oracle.IP:
        d = -(d64 @ q64)
    else:
        nd = np.linalg.norm(d64, axis=1)
        nq = np.linalg.norm(q64)
        d = 1.0 - (d64 @ q64) / (nd * nq)
    d = d.astype(np.float32)
    order = np.lexsort((np.arange(len(d)), d))
    return order[:K].astype(np.int32), d[order[:K]]


def ring_plus_random_graph(n, deg, rng):
    adj = np.full((n, deg), -1, np.int32)
    for v in range(n):
        adj[v, 0] = (v + 1) % n
        adj[v, 1:] = rng.integers(0, n, deg - 1)
    return adj


@pytest.mark.parametrize("metric", [oracle.L2, oracle.IP, oracle.COSINE])
@pytest.mark.parametrize("flags", [oracle.PLAIN, oracle.OPTIMIZED])
def test_full_queue_is_exact_knn(metric, flags):
    """P4: with L >= n on a graph where every vertex is reachable from the
    entry, Algorithm 1 expands every vertex, so topk is the exact top-L."""
    rng = np.random.default_rng(7)
    n, dim, deg, K = 60, 5, 4, 10
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = ring_plus_random_graph(n, deg, rng)
    qs = rng.standard_normal((8, dim)).astype(np.float32)
    ids, dists, _, capped = oracle.search(data, adj, qs, K, n, metric=metric, flags=flags)
    assert capped == 0
    for i in range(len(qs)):
        ti, td = numpy_topk(data, qs[i], K, metric)
        np.testing.assert_array_equal(ids[i], ti)
        np.testing.assert_allclose(dists[i], td, rtol=1e-6, atol=1e-6)
    bi, bd = oracle.bruteforce(data, qs, K, metric)
    np.testing.assert_array_equal(bi, ids)


@pytest.mark.parametrize("L", [10, 11, 16, 40])
def test_complete_graph_exact_for_any_L(L):
    """P4: on a complete graph every vertex is a candidate of the first
    expansion, so any L >= K returns the exact top-K."""
    rng = np.random.default_rng(11)
    n, dim, K = 40, 3, 10
    data = rng.integers(-5, 6, (n, dim)).astype(np.float32)  # many exact ties
    adj = np.array([[u for u in range(n) if u != v] for v in range(n)], np.int32)
    qs = rng.integers(-5, 6, (20, dim)).astype(np.float32)
    ids, dists, _, _ = oracle.search(data, adj, qs, K, L)
    for i in range(len(qs)):
        ti, td = numpy_topk(data, qs[i], K, oracle.L2)
        np.testing.assert_array_equal(ids[i], ti)
        np.testing.assert_array_equal(dists[i], td)


def greedy_descent(data, adj, q, entry=0):
    """NSW greedy search [46]: move to the best neighbour while it improves."""
    def key(v):
        return (float(np.float32(((data[v].astype(np.float64) - q) ** 2).sum())), v)
    cur = entry
    while True:
        nb = [int(v) for v in adj[cur] if v >= 0]
        best = min(nb, key=key) if nb else None
        if best is None or key(best) >= key(cur):
            return cur
        cur = best


def test_L1_is_greedy_descent():
    """P5: L = K = 1 reduces Algorithm 1 (+ all optimizations) to greedy descent."""
    rng = np.random.default_rng(3)
    n, dim, deg = 200, 4, 6
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    qs = rng.standard_normal((50, dim)).astype(np.float32)
    for flags in (oracle.PLAIN, oracle.OPTIMIZED):
        ids, _, _, _ = oracle.search(data, adj, qs, 1, 1, flags=flags)
        for i in range(len(qs)):
            assert ids[i, 0] == greedy_descent(data, adj, qs[i].astype(np.float64))


def test_padding_and_repeats_and_short_results():
    """R6: -1 is padding, a repeated id is located once; fewer than K
    reachable vertices pad the output with (-1, +inf)."""
    data = np.array([[0.0], [1.0], [2.0], [3.0], [9.0]], np.float32)
    adj = np.array([[1, 1, -1, 2], [0, 2, 2, -1], [1, -1, -1, -1],
                    [4, -1, -1, -1], [3, -1, -1, -1]], np.int32)
    ids, dists, ctr, _ = oracle.search(data, adj, np.array([[0.5]], np.float32), 5, 8,
                                       flags=oracle.PLAIN)
    assert ids[0].tolist() == [0, 1, 2, -1, -1]
    assert np.isinf(dists[0, 3:]).all()
    assert ctr[0, 0] == 3  # 0, then 1 and 2 once each


def test_recall_definition():
    """Recall(A) = |A ∩ B| / |B|, averaged over queries."""
    assert oracle.recall([[1, 2, 3]], [[3, 4, 5]]) == pytest.approx(1 / 3)
    assert oracle.recall([[1, 2], [5, 6]], [[1, 2], [7, 8]]) == pytest.approx(0.5)


def test_merge_shards_definition():
    """P:471 "merge the results": K smallest (dist, id) over all shards, ties
    by id, padding (-1, inf) ignored; worked by hand."""
    ids = [np.array([[5, 9, -1]]), np.array([[2, 7, 8]])]
    d = [np.array([[1.0, 3.0, np.inf]], np.float32), np.array([[1.0, 2.0, 9.0]], np.float32)]
    i, dd = oracle.merge_shards(ids, d, 4)
    assert i.tolist() == [[2, 5, 7, 9]]
    assert dd.tolist() == [[1.0, 1.0, 2.0, 3.0]]
    i, dd = oracle.merge_shards([np.array([[-1, -1]])], [np.full((1, 2), np.inf, np.float32)], 2)
    assert i.tolist() == [[-1, -1]] and np.isinf(dd).all()
