"""Pins of the oracle's multi-step probing (§V; reading R13), CPU only.

* a hand-worked trace on the Fig. 1 toy with 2 pops per iteration
  (tests/golden/multistep_toy.txt);
* steps = 1 is Algorithm 1 (the existing pins then cover it);
* L = 1: the second pop can never beat a full topk, so every width is the
  greedy search;
* full queue on a connected graph: exact brute-force kNN for every width;
* the §IV optimizations still leave the result unchanged (Observation 1,
  P:431 and P:435 hold pop by pop), with integer ties.
"""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle
from _golden import golden_path
import test_oracle_pins as pins
import test_oracle_equiv as equiv


def load_golden():
    states, result, counters = {}, None, None
    with open(golden_path("multistep_toy.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            if line.startswith("steps2"):
                head, q, t, vis = [s.strip() for s in line.split("|")]
                parse = lambda s: [] if s == "-" else [int(x) for x in s.split()]
                states[int(head.split()[1])] = (parse(q), parse(t), parse(vis))
            elif line.startswith("result"):
                result = [int(x) for x in line.split()[1:]]
            elif line.startswith("counters"):
                counters = [int(x) for x in line.split()[1:]]
    return states, result, counters


def test_hand_worked_two_step_trace():
    data, adj, _, _ = pins.load_toy()
    states, result, counters = load_golden()
    seen = {}

    def cb(it, q, t, vis):
        seen[it] = ([x + 1 for x in q], [x + 1 for x in t], [x + 1 for x in vis])

    ids, _, ctr, capped = oracle.search(data, adj, np.zeros((1, 1), np.float32), 3, 3,
                                        flags=oracle.PLAIN, trace=cb, steps=2)
    assert capped == 0
    assert seen == states
    assert [int(x) + 1 for x in ids[0]] == result
    assert ctr[0].tolist() == counters


def _graph(n, deg, rng, connected=True):
    adj = rng.integers(-1, n, (n, deg)).astype(np.int32)
    if connected:
        adj[:, 0] = (np.arange(n) + 1) % n
    return adj


def test_steps1_is_algorithm1():
    rng = np.random.default_rng(0)
    data = rng.standard_normal((200, 4)).astype(np.float32)
    adj = _graph(200, 6, rng)
    qs = rng.standard_normal((20, 4)).astype(np.float32)
    a = oracle.search(data, adj, qs, 5, 16)
    b = oracle.search(data, adj, qs, 5, 16, steps=1)
    for x, y in zip(a[:3], b[:3]):
        np.testing.assert_array_equal(x, y)


@pytest.mark.parametrize("steps", [2, 3, 4])
def test_queue_of_one_is_greedy_for_every_width(steps):
    rng = np.random.default_rng(steps)
    data = rng.standard_normal((300, 3)).astype(np.float32)
    adj = _graph(300, 5, rng)
    qs = rng.standard_normal((30, 3)).astype(np.float32)
    a = oracle.search(data, adj, qs, 1, 1)
    b = oracle.search(data, adj, qs, 1, 1, steps=steps)
    for x, y in zip(a[:3], b[:3]):
        np.testing.assert_array_equal(x, y)


@pytest.mark.parametrize("steps", [2, 3, 4])
def test_full_queue_is_exact(steps):
    rng = np.random.default_rng(10 + steps)
    n = 150
    data = rng.integers(0, 8, (n, 2)).astype(np.float32)  # many ties
    adj = _graph(n, 4, rng)
    qs = rng.integers(0, 8, (25, 2)).astype(np.float32)
    ids, d, _, capped = oracle.search(data, adj, qs, 7, n + 5, steps=steps)
    bi, bd = oracle.bruteforce(data, qs, 7)
    assert capped == 0
    np.testing.assert_array_equal(ids, bi)
    np.testing.assert_array_equal(d, bd)


@settings(max_examples=300, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(equiv.problems(), st.integers(2, 4))
def test_optimizations_preserve_multistep_result(prob, steps):
    data, adj, qs, K, L, entry = prob
    ref = oracle.search(data, adj, qs, K, L, flags=oracle.PLAIN, entry=entry, steps=steps)
    assert ref[3] == 0
    for flags in equiv.MODES:
        got = oracle.search(data, adj, qs, K, L, flags=flags, entry=entry, steps=steps,
                            max_iters=100000)
        assert got[3] == 0
        np.testing.assert_array_equal(got[0], ref[0])
        np.testing.assert_array_equal(got[1], ref[1])
        # the popped sequence is the same, so are the expansions
        np.testing.assert_array_equal(got[2][:, 1], ref[2][:, 1])
