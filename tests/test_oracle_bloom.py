"""P7: the Bloom-filter visited set of §IV-B, CPU only."""
import numpy as np

import oracle


def test_bloom_no_false_negatives_and_paper_fpr():
    """"a Bloom filter with around 300 32-bit integers has less than 1% false
    positives when inserting 1,000 vertices".  With k = 7 (reading A11)
    theory gives (1 - e^{-7000/9600})^7 = 0.997 %."""
    rng = np.random.default_rng(0)
    ids = rng.choice(10_000_000, 201_000, replace=False).astype(np.int32)
    ins, probe = ids[:1000], ids[1000:]
    member = oracle.bloom_probe(300 * 32, ins, ins)
    assert member.all(), "no false negatives"
    fpr = oracle.bloom_probe(300 * 32, ins, probe).mean()
    theory = (1 - np.exp(-7 * 1000 / 9600)) ** 7
    assert abs(theory - 0.00997) < 1e-4
    assert fpr < 0.011  # 200k probes: sd = 0.022 %
    assert fpr > 0.0085


def test_bloom_power_of_two_default_size():
    """The product's default m = 2^ceil(log2(80 L)) bits keeps the FPR far below
    1 % at 8L inserts."""
    rng = np.random.default_rng(1)
    for L in (16, 64, 256):
        m = oracle.default_bloom_bits(L)
        assert m & (m - 1) == 0 and m >= 80 * L
        ids = rng.choice(50_000_000, 8 * L + 100_000, replace=False).astype(np.int32)
        ins, probe = ids[:8 * L], ids[8 * L:]
        assert oracle.bloom_probe(m, ins, ins).all()
        assert oracle.bloom_probe(m, ins, probe).mean() < 0.003


def test_bloom_search_equals_plain_without_false_positives():
    """With a filter so large that false positives are negligible, bounded q +
    selected insertion with a Bloom visited set returns Algorithm 1's result
    (deletion is off: a Bloom filter cannot delete)."""
    rng = np.random.default_rng(2)
    n, dim, deg = 400, 6, 8
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    qs = rng.standard_normal((20, dim)).astype(np.float32)
    ref = oracle.search(data, adj, qs, 10, 24, flags=oracle.PLAIN)
    blm = oracle.search(data, adj, qs, 10, 24, flags=oracle.OPTIMIZED_BLOOM,
                        bloom_bits=1 << 26)
    np.testing.assert_array_equal(ref[0], blm[0])
    np.testing.assert_array_equal(ref[1], blm[1])


def test_tiny_bloom_loses_recall_not_correctness():
    """A saturated filter only skips vertices (false positives): output stays
    sorted, unique and a subset of real vertices, and never computes more
    distances than the exact-set run."""
    rng = np.random.default_rng(4)
    n, dim, deg = 400, 6, 8
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    qs = rng.standard_normal((20, dim)).astype(np.float32)
    ex = oracle.search(data, adj, qs, 10, 24, flags=oracle.BOUNDED_Q | oracle.SEL)
    ids, d, ctr, _ = oracle.search(data, adj, qs, 10, 24, flags=oracle.OPTIMIZED_BLOOM,
                                   bloom_bits=64)
    assert (ctr[:, 0] <= ex[2][:, 0]).all()
    for i in range(len(qs)):
        v = ids[i][ids[i] >= 0]
        assert len(set(v.tolist())) == len(v)
        assert (np.diff(d[i][ids[i] >= 0]) >= 0).all()
