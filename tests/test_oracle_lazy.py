"""Pins of the lazy visited-deletion schedule (reading R14, a schedule of
§IV-E), CPU only: any capacity C >= 2L + 32 gives Algorithm 1's result
and the same expansions (the popped sequence cannot change); C = infinity is
exactly hashtable-sel (no deletion, Fig. 7), counters included; |visited|
never exceeds C after an iteration."""
import numpy as np
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle
import test_oracle_equiv as equiv


@settings(max_examples=300, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(equiv.problems(), st.integers(0, 40))
def test_lazy_schedule_preserves_result(prob, extra):
    data, adj, qs, K, L, entry = prob
    ref = oracle.search(data, adj, qs, K, L, flags=oracle.PLAIN, entry=entry)
    eager = oracle.search(data, adj, qs, K, L, flags=oracle.OPTIMIZED, entry=entry)
    cap = 2 * L + 32 + extra
    lazy = oracle.search(data, adj, qs, K, L, flags=oracle.OPTIMIZED_LAZY, lazy_cap=cap,
                         entry=entry)
    np.testing.assert_array_equal(lazy[0], ref[0])
    np.testing.assert_array_equal(lazy[1], ref[1])
    np.testing.assert_array_equal(lazy[2][:, 1], eager[2][:, 1])


def test_unbounded_capacity_is_hashtable_sel():
    rng = np.random.default_rng(7)
    for trial in range(20):
        n, dim, deg = 400, 4, 8
        data = rng.integers(0, 9, (n, dim)).astype(np.float32)
        adj = rng.integers(-1, n, (n, deg)).astype(np.int32)
        qs = rng.integers(0, 9, (10, dim)).astype(np.float32)
        L = int(rng.integers(1, 48))
        a = oracle.search(data, adj, qs, 1, L, flags=oracle.OPTIMIZED_LAZY, lazy_cap=10 ** 9)
        b = oracle.search(data, adj, qs, 1, L, flags=oracle.HASHTABLE_SEL)
        for x, y in zip(a[:3], b[:3]):
            np.testing.assert_array_equal(x, y)


def test_visited_stays_within_capacity():
    rng = np.random.default_rng(8)
    n, dim, deg = 2000, 6, 16
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    q = rng.standard_normal((1, dim)).astype(np.float32)
    for L in (4, 16, 40):
        cap = 2 * L + 32
        sizes = []
        oracle.search(data, adj, q, 4, L, flags=oracle.OPTIMIZED_LAZY, lazy_cap=cap,
                      trace=lambda it, qq, t, vis: sizes.append(len(vis)))
        assert max(sizes) <= cap
        assert max(sizes) > 2 * L  # the deferral actually happened


def test_lazy_recomputes_less_on_a_navigable_graph():
    """What the schedule is for: on an NSW-like graph it computes fewer
    distances than eager deletion at the same result."""
    from workloads.graph import build_graph
    from workloads.synth import gauss
    x = gauss(4000, 16, 3)
    adj = build_graph(x, degree=16).numpy()
    xn = x.numpy()
    q = gauss(50, 16, 4).numpy()
    L = 32
    e = oracle.search(xn, adj, q, 10, L, flags=oracle.OPTIMIZED)
    z = oracle.search(xn, adj, q, 10, L, flags=oracle.OPTIMIZED_LAZY, lazy_cap=512)
    np.testing.assert_array_equal(e[0], z[0])
    assert z[2][:, 0].sum() < 0.9 * e[2][:, 0].sum()
