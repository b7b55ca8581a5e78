"""Reading R17 (the bounded union: q and topk kept as one list W of the L
best discovered keys with a popped mark), CPU only.

Pinned against Algorithm 1 itself (the PLAIN mode: unbounded q, exact visited
set never deleted from, topk bounded at L — P:41-49), not against the
optimized modes: the union must return the same ids and distances and pop the
same sequence (n_exp), on graphs with integer coordinates so that exact
distance ties exercise the (dist, id) order (R2)."""
import numpy as np
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle
import test_oracle_pins as pins

UNION_MODES = [oracle.OPTIMIZED_UNION, oracle.BOUNDED_Q | oracle.SEL | oracle.UNION,
               oracle.BOUNDED_Q | oracle.UNION]


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
    cap = draw(st.integers(L + 32, 2 * L + 80))
    return data, adj, qs, K, L, entry, cap


@settings(max_examples=400, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(problems())
def test_union_equals_algorithm_1(prob):
    data, adj, qs, K, L, entry, cap = prob
    ids0, d0, c0, _ = oracle.search(data, adj, qs, K, L, flags=oracle.PLAIN, entry=entry)
    for flags, kw in [(m, {}) for m in UNION_MODES] + [
            (oracle.OPTIMIZED_UNION_LAZY, {"lazy_cap": cap})]:
        ids, d, c, capped = oracle.search(data, adj, qs, K, L, flags=flags, entry=entry,
                                          max_iters=100000, **kw)
        assert capped == 0
        np.testing.assert_array_equal(ids, ids0)
        np.testing.assert_array_equal(d, d0)
        np.testing.assert_array_equal(c[:, 1], c0[:, 1])  # the same popped sequence


def test_union_larger_float_graphs():
    rng = np.random.default_rng(321)
    for trial in range(20):
        n, dim, deg = 400, 4, 8
        data = rng.standard_normal((n, dim)).astype(np.float32)
        adj = rng.integers(0, n, (n, deg)).astype(np.int32)
        qs = rng.standard_normal((8, dim)).astype(np.float32)
        L = int(rng.integers(4, 160))
        K = int(rng.integers(1, L + 1))
        ref = oracle.search(data, adj, qs, K, L, flags=oracle.PLAIN)
        un = oracle.search(data, adj, qs, K, L, flags=oracle.OPTIMIZED_UNION)
        lz = oracle.search(data, adj, qs, K, L, flags=oracle.OPTIMIZED_UNION_LAZY,
                           lazy_cap=L + 32)
        for o in (un, lz):
            np.testing.assert_array_equal(o[0], ref[0])
            np.testing.assert_array_equal(o[1], ref[1])
            np.testing.assert_array_equal(o[2][:, 1], ref[2][:, 1])


def test_union_fig1_toy():
    """Fig. 1: the toy returns {2, 7, 8} with 4 expansions; eager
    deletion under the union recomputes nothing the separate structures keep
    here (W holds q ∪ topk whenever |q ∪ topk| <= L)."""
    data, adj, _, result = pins.load_toy()
    q = np.zeros((1, 1), np.float32)
    ids, _, c, _ = oracle.search(data, adj, q, 3, 3, flags=oracle.OPTIMIZED_UNION)
    assert [int(x) + 1 for x in ids[0]] == result
    assert c[0, 1] == 4


def test_union_full_queue_is_exact():
    """P4 for R17: with L >= n on a connected graph every vertex is reached and
    the result is the brute-force top-K."""
    rng = np.random.default_rng(8)
    n, dim = 120, 3
    data = rng.integers(0, 9, (n, dim)).astype(np.float32)
    adj = np.stack([(np.arange(n) + s) % n for s in (1, n - 1, 7)], 1).astype(np.int32)
    qs = rng.integers(0, 9, (5, dim)).astype(np.float32)
    ids, d, _, _ = oracle.search(data, adj, qs, 10, n, flags=oracle.OPTIMIZED_UNION)
    bi, bd = oracle.bruteforce(data, qs, 10)
    np.testing.assert_array_equal(ids, bi)
    np.testing.assert_array_equal(d, bd)
