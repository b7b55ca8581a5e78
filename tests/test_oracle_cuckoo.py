"""Reading R10: the Cuckoo-filter visited set (ref [14]), CPU only.

Pinned by what the data structure guarantees: no false negatives while nothing
is deleted and nothing is dropped, a false-positive rate below the
2·4/2^16 bound of 16-bit fingerprints in 4-slot buckets, deletion of one copy,
and - with a filter large enough that false positives are negligible - the
search reduces to the exact optimized search (bounded q + sel + del)."""
import numpy as np

import oracle


def test_cuckoo_no_false_negatives_and_fpr_bound():
    rng = np.random.default_rng(0)
    buckets = 1 << 12                       # 16384 slots
    ids = rng.choice(1 << 30, 8192 + 400_000, replace=False)
    ins, probe = ids[:8192], ids[8192:]     # 50 % load
    member, drops = oracle.cuckoo_probe(buckets, ins, ins)
    assert drops == 0 and member.all()
    fp, _ = oracle.cuckoo_probe(buckets, ins, probe)
    bound = 2 * 4 / 2 ** 16                 # two buckets x four 16-bit slots
    assert fp.mean() < bound
    # a nearly full table (95 %) still holds everything (kicks relocate)
    ins95 = ids[:int(0.95 * 4 * buckets)]
    member, drops = oracle.cuckoo_probe(buckets, ins95, ins95)
    assert drops == 0 and member.all()


def test_cuckoo_deletion_removes_one_copy():
    rng = np.random.default_rng(1)
    ids = rng.choice(1 << 30, 2000, replace=False)
    a, b = ids[:1000], ids[1000:]
    ops = np.concatenate([a, b, -(a + 1)])  # insert a and b, erase a
    seen, drops = oracle.cuckoo_probe(1 << 10, ops, np.concatenate([a, b]))
    assert drops == 0
    assert seen[1000:].all(), "erasing a must not remove b"
    assert seen[:1000].mean() < 0.01, "a is gone (up to fingerprint collisions)"
    # inserting an id twice and erasing once leaves one copy
    x = np.array([12345, 12345, -12346])
    seen, _ = oracle.cuckoo_probe(64, x, np.array([12345]))
    assert seen.all()


def test_cuckoo_search_reduces_to_exact_when_large():
    rng = np.random.default_rng(2)
    n, dim, deg = 500, 6, 8
    data = rng.integers(0, 10, (n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    qs = rng.integers(0, 10, (40, dim)).astype(np.float32)
    for L in (4, 16, 40):
        ex = oracle.search(data, adj, qs, 4, L, flags=oracle.OPTIMIZED)
        ck = oracle.search(data, adj, qs, 4, L, flags=oracle.OPTIMIZED_CUCKOO,
                           bloom_bits=1 << 14)
        np.testing.assert_array_equal(ex[0], ck[0])
        np.testing.assert_array_equal(ex[2], ck[2])


def test_fig7_variants_keep_algorithm1_result():
    """hashtable / hashtable-sel / hashtable-sel-del (Fig. 7) are exact
    visited sets: all return Algorithm 1's result."""
    rng = np.random.default_rng(3)
    n, dim, deg = 400, 5, 8
    data = rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(0, n, (n, deg)).astype(np.int32)
    qs = rng.standard_normal((30, dim)).astype(np.float32)
    ref = oracle.search(data, adj, qs, 10, 32, flags=oracle.PLAIN)
    for f in (oracle.HASHTABLE, oracle.HASHTABLE_SEL, oracle.OPTIMIZED):
        got = oracle.search(data, adj, qs, 10, 32, flags=f)
        np.testing.assert_array_equal(ref[0], got[0])
