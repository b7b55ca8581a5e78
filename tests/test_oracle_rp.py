"""Pins of the oracle's 1-bit random projection (§VII) and its
Hamming-distance search (readings R11, R12) against what the paper and the
mathematics fix (CPU only).

* a hand-worked code (layout, sign, packing: a transposed R, a flipped sign or
  an MSB-first packing each fail it);
* the collision law Pr[sgn<u,r> = sgn<v,r>] = 1 - theta/pi;
* Hamming closed forms against an independent bit count (np.unpackbits);
* Table IV's sizes and "more than 190 times smaller";
* search over codes: full queue == brute force, plain == optimized with the
  integer distances' many ties, sign/scale invariances of the codes.
"""
import math

import numpy as np
import pytest

import oracle
from _golden import golden_path


def test_hand_worked_code():
    # x = (2, -1); r_0 = (1, 0) -> 2 > 0; r_1 = (0, 1) -> -1; r_2 = (1, 1) -> 1;
    # r_3 = (1, -1) -> 3; r_32 = (-1, 0) -> -2; r_33 = (0, -1) -> 1
    R = np.zeros((64, 2), np.float32)
    R[0], R[1], R[2], R[3] = (1, 0), (0, 1), (1, 1), (1, -1)
    R[32], R[33] = (-1, 0), (0, -1)
    c = oracle.rp_encode(np.array([[2.0, -1.0]], np.float32), R)
    assert c.shape == (1, 2) and c.dtype == np.uint32
    assert int(c[0, 0]) == 0b1101  # bits 0, 2, 3
    assert int(c[0, 1]) == 0b10    # bit 33 -> word 1, position 1


def test_sign_of_zero_is_bit_zero():
    R = np.random.default_rng(0).standard_normal((64, 5)).astype(np.float32)
    assert not oracle.rp_encode(np.zeros((1, 5), np.float32), R).any()
    # a projection that cancels exactly: <(1, 1), (1, -1)> = 0
    R2 = np.zeros((32, 2), np.float32)
    R2[0] = (1, -1)
    R2[1] = (1, -0.5)
    assert int(oracle.rp_encode(np.array([[1.0, 1.0]], np.float32), R2)[0, 0]) == 0b10


def test_invariances():
    rng = np.random.default_rng(1)
    x = rng.standard_normal((50, 16)).astype(np.float32)
    R = rng.standard_normal((96, 16)).astype(np.float32)
    c = oracle.rp_encode(x, R)
    np.testing.assert_array_equal(oracle.rp_encode(x * 3.0, R), c)       # sgn(c<x,r>) for c > 0
    np.testing.assert_array_equal(oracle.rp_encode(-x, R), ~c)           # no zero projections here
    np.testing.assert_array_equal(oracle.rp_encode(x, -R), ~c)


@pytest.mark.parametrize("theta", [0.3, 1.0, math.pi / 2, 2.5])
def test_collision_probability(theta):
    """Pr(sgn<u,r> = sgn<v,r>) = 1 - theta(u,v)/pi, r iid N(0,1)."""
    rng = np.random.default_rng(int(theta * 1000))
    d, h = 48, 32 * 256
    Q, _ = np.linalg.qr(rng.standard_normal((d, 2)))
    u = Q[:, 0]
    v = math.cos(theta) * Q[:, 0] + math.sin(theta) * Q[:, 1]
    R = rng.standard_normal((h, d)).astype(np.float32)
    c = oracle.rp_encode(np.stack([u, v]).astype(np.float32), R)
    agree = 1.0 - oracle.hamming(c[0], c[1]) / h
    p = 1.0 - theta / math.pi
    assert abs(agree - p) < 4.5 * math.sqrt(p * (1 - p) / h) + 1e-3


def test_hamming_closed_forms():
    rng = np.random.default_rng(2)
    for words in (1, 2, 4, 16):
        a = rng.integers(0, 2**32, words, dtype=np.uint64).astype(np.uint32)
        b = rng.integers(0, 2**32, words, dtype=np.uint64).astype(np.uint32)
        ref = int(np.unpackbits((a ^ b).view(np.uint8)).sum())
        assert oracle.hamming(a, b) == ref == oracle.hamming(b, a)
        assert oracle.hamming(a, a) == 0
        assert oracle.hamming(a, ~a) == 32 * words
        one = a.copy()
        one[words - 1] ^= np.uint32(1 << 31)
        assert oracle.hamming(a, one) == 1


def test_table4_sizes():
    rows = []
    with open(golden_path("table4_hashed_sizes.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].split()
            if line:
                rows.append(line)
    mib = 1 << 20
    for bits, n, mb in rows:
        n, mb = int(n), int(mb)
        if bits == "original":
            orig = n * 784 * 4 / mib
            assert round(orig / 1000) == mb // 1000  # "2.4 x 10^4"
        else:
            assert math.ceil(oracle.code_bytes(n, int(bits)) / mib) == mb
    # "128-bit hashing makes the original dataset more than 190 times smaller"
    assert (8_090_000 * 784 * 4) / oracle.code_bytes(8_090_000, 128) > 190


def _rand_graph(n, deg, rng):
    adj = np.full((n, deg), -1, np.int32)
    for v in range(n):
        k = rng.integers(1, deg + 1)
        adj[v, :k] = rng.choice(n, k, replace=False)
    # a ring keeps everything reachable from the entry
    adj[:, 0] = (np.arange(n) + 1) % n
    return adj


def test_hamming_search_full_queue_is_exact():
    rng = np.random.default_rng(3)
    n, words = 300, 2
    codes = rng.integers(0, 2**32, (n, words), dtype=np.uint64).astype(np.uint32)
    q = rng.integers(0, 2**32, (20, words), dtype=np.uint64).astype(np.uint32)
    adj = _rand_graph(n, 8, rng)
    ids, dists, _, capped = oracle.search_codes(codes, adj, q, 10, n)
    bi, bd = oracle.bruteforce_codes(codes, q, 10)
    assert capped == 0
    np.testing.assert_array_equal(ids, bi)
    np.testing.assert_array_equal(dists, bd)
    # distances are integers and equal the independent bit count
    for r in range(len(q)):
        for j in range(10):
            ref = int(np.unpackbits((q[r] ^ codes[ids[r, j]]).view(np.uint8)).sum())
            assert dists[r, j] == ref


@pytest.mark.parametrize("L", [4, 10, 32])
def test_hamming_plain_equals_optimized(L):
    """Observation 1 / P:431 / P:435 hold for the Hamming keys (many ties)."""
    rng = np.random.default_rng(L)
    n = 400
    codes = rng.integers(0, 2**32, (n, 1), dtype=np.uint64).astype(np.uint32)
    codes &= np.uint32(0x0000ffff)  # 16 live bits: ties everywhere
    q = rng.integers(0, 2**16, (30, 1), dtype=np.uint64).astype(np.uint32)
    adj = _rand_graph(n, 6, rng)
    a = oracle.search_codes(codes, adj, q, 4, L, flags=oracle.PLAIN)
    b = oracle.search_codes(codes, adj, q, 4, L, flags=oracle.OPTIMIZED)
    np.testing.assert_array_equal(a[0], b[0])
    np.testing.assert_array_equal(a[1], b[1])


def test_codes_track_the_original_neighbours():
    """Fig. 14's premise: more bits estimate the angle better, so the
    Hamming top-1 agrees with the original top-1 more often as h grows."""
    from workloads import synth
    gen = synth.MnistLike(784, 600)
    x = gen.sample(3000, 600).numpy()
    q = gen.sample(40, 601).numpy()
    truth, _ = oracle.bruteforce(x, q, 1, nthreads=4)
    hits = []
    for h in (32, 512):
        R = synth.rp_matrix(h, 784, 603).numpy()
        bi, _ = oracle.bruteforce_codes(oracle.rp_encode(x, R, nthreads=4),
                                        oracle.rp_encode(q, R), 5, nthreads=4)
        hits.append(np.mean([truth[i, 0] in bi[i] for i in range(len(q))]))
    assert hits[1] > hits[0] and hits[1] >= 0.6


def test_rp_recipe_is_exact_in_fp32():
    """The workload's R (workloads.synth.rp_matrix) and integer pixels keep every
    partial sum of every projection a multiple of 1/64 below 2^24 / 64, so the
    fp64 oracle and any fp32 summation order decide the same sign."""
    from workloads import synth
    gen = synth.MnistLike(784, 600)
    x = gen.sample(2000, 600).double()
    R = synth.rp_matrix(512, 784, 603).double()
    k = R * 64
    assert bool((k == k.round()).all()) and float(k.abs().max()) <= 256
    assert bool((x == x.round()).all())
    assert float((x.abs() @ k.abs().T).max()) < 2 ** 24
