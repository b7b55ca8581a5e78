"""P3 (equivalence of the §IV optimizations) and P6 (invariants), CPU only.

Observation 1, selected insertion and visited deletion
 claim to leave Algorithm 1's output unchanged.  Integer coordinates
make exact distance ties common, which exercises the (dist, id) order (R2).
"""
import numpy as np
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle

MODES = [oracle.BOUNDED_Q, oracle.BOUNDED_Q | oracle.SEL, oracle.OPTIMIZED,
         oracle.BOUNDED_Q | oracle.DEL]


@st.composite
def problems(draw):
    n = draw(st.integers(2, 40))
    deg = draw(st.integers(1, 6))
    dim = draw(st.integers(1, 3))
    seed = draw(st.integers(0, 2 ** 31 - 1))
    rng = np.random.default_rng(seed)
    data = rng.integers(0, 6, (n, dim)).astype(np.float32)
    adj = rng.integers(-1, n, (n, deg)).astype(np.int32)
    qs = rng.integers(0, 6, (3, dim)).astype(np.float32)
    L = draw(st.integers(1, n + 2))
    K = draw(st.integers(1, L))
    entry = draw(st.integers(0, n - 1))
    return data, adj, qs, K, L, entry


@settings(max_examples=400, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(problems())
def test_optimizations_preserve_result(prob):
    data, adj, qs, K, L, entry = prob
    ids0, d0, c0, cap0 = oracle.search(data, adj, qs, K, L, flags=oracle.PLAIN, entry=entry)
    assert cap0 == 0
    for flags in MODES:
        ids, d, c, cap = oracle.search(data, adj, qs, K, L, flags=flags, entry=entry,
                                       max_iters=100000)
        assert cap == 0, "terminates"
        np.testing.assert_array_equal(ids, ids0)
        np.testing.assert_array_equal(d, d0)


def test_optimizations_preserve_result_larger_graphs():
    rng = np.random.default_rng(123)
    for trial in range(30):
        n, dim, deg = 300, 4, 8
        data = rng.standard_normal((n, dim)).astype(np.float32)
        adj = rng.integers(0, n, (n, deg)).astype(np.int32)
        qs = rng.standard_normal((10, dim)).astype(np.float32)
        L = int(rng.integers(4, 64))
        K = int(rng.integers(1, L + 1))
        ref = oracle.search(data, adj, qs, K, L, flags=oracle.PLAIN)
        opt = oracle.search(data, adj, qs, K, L, flags=oracle.OPTIMIZED)
        np.testing.assert_array_equal(ref[0], opt[0])
        # the optimizations trade memory for recomputation: never fewer distances
        assert (opt[2][:, 0] >= ref[2][:, 0]).all()
        # ... and the same expansions (the popped sequence is identical)
        np.testing.assert_array_equal(opt[2][:, 1], ref[2][:, 1])


@settings(max_examples=200, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(problems())
def test_invariants_under_sel_del(prob):
    """P6: |q| <= L, |topk| <= L, visited == q ∪ topk (so <= 2L), no id
    twice in q ∪ topk, topk's max never increases once full."""
    data, adj, qs, K, L, entry = prob
    dist = lambda v: float(((data[v].astype(np.float64) - qs[0]) ** 2).sum())
    key = lambda v: (np.float32(dist(v)), v)
    state = {"prev_max": None}

    def cb(it, q, t, vis):
        assert len(q) <= L and len(t) <= L
        both = q + t
        assert len(set(both)) == len(both)
        assert sorted(vis) == sorted(both)
        assert [key(v) for v in q] == sorted(key(v) for v in q)
        assert [key(v) for v in t] == sorted(key(v) for v in t)
        if len(t) == L:
            m = key(t[-1])
            if state["prev_max"] is not None:
                assert m <= state["prev_max"]
            state["prev_max"] = m

    ids, d, _, _ = oracle.search(data, adj, qs[:1], K, L, flags=oracle.OPTIMIZED,
                                 entry=entry, trace=cb)
    valid = ids[0] >= 0
    keys = [(d[0, i], ids[0, i]) for i in range(K) if valid[i]]
    assert keys == sorted(keys)
    assert len(set(ids[0][valid])) == valid.sum()


def test_counters_plain_mode_count_each_visited_once():
    """In plain mode each vertex enters visited exactly once, when its distance
    is computed (Alg. 1 lines 11-12), so n_dist == |visited| at the end."""
    rng = np.random.default_rng(5)
    n, dim, deg = 500, 8, 10
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    q = rng.standard_normal((1, dim)).astype(np.float32)
    last = {}

    def cb(it, qq, t, vis):
        last["vis"] = vis
        last["it"] = it

    _, _, ctr, _ = oracle.search(data, adj, q, 10, 32, flags=oracle.PLAIN, trace=cb)
    assert ctr[0, 0] == len(last["vis"])
    assert ctr[0, 1] == last["it"]
