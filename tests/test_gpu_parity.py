"""GPU parity: the CUDA path (through the C ABI) against the oracle.

Bars (BASELINE.json north_star):
 * integer-valued data (pin P8): ids, distances AND counters bit-exact for
   every query;
 * float data: top-K ids identical on >= 99.5 % of queries, distances within
   rtol 1e-5 + atol 1e-5 * scale, recall within 0.002 of the oracle's.
"""
import ctypes

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from workloads.graph import build_graph  # noqa: E402
from workloads.synth import CONFIGS, make_data  # noqa: E402

from _golden import golden_path  # noqa: E402
import test_oracle_pins as pins  # noqa: E402


def song():
    from paper_conf_icde_zhaotl20_b200 import song as s
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return s


ORACLE_FLAGS = {"hash": oracle.OPTIMIZED, "bloom": oracle.OPTIMIZED_BLOOM,
                "hashtable": oracle.HASHTABLE, "hashtable-sel": oracle.HASHTABLE_SEL,
                "cuckoo": oracle.OPTIMIZED_CUCKOO}
ALL_VISITED = list(ORACLE_FLAGS)


def lazy_cap_for(L, dim=128, metric="l2"):
    """The lazy-deletion capacity the library uses for visited_cap = 0, read
    from its own plan (song_search_plan_get) — never re-derived here."""
    return song_plan_cap(L, dim, metric)


def song_plan_cap(L, dim, metric):
    from paper_conf_icde_zhaotl20_b200 import song as s
    return s.default_visited_cap(L, dim, metric)


def oracle_kw(visited, L, steps=1, visited_cap=0, log2=0, queue_kind="auto", idx=None):
    """The oracle mode matching a GPU search, read from the library's plan
    (song_search_plan_get): the hash's deletion schedule is lazy (reading
    R14) unless visited_cap = -1 or steps > 1 (eager), and queues above 128
    (or queue_kind="union") are the bounded union of reading R17."""
    from paper_conf_icde_zhaotl20_b200 import song as s
    kw = dict(flags=ORACLE_FLAGS[visited], bloom_bits=bloom_bits_for(L, log2, visited))
    if visited == "hash":
        prm = s.Params(K=1, queue_len=L, steps=steps, visited_cap=visited_cap,
                       queue_kind=queue_kind)
        pl = idx.plan(prm) if idx is not None else s.plan(prm, 128)
        flags = oracle.OPTIMIZED
        if pl.visited_cap > 0:
            flags |= oracle.LAZY
            kw["lazy_cap"] = pl.visited_cap
        if pl.queue_kind == 2:
            flags |= oracle.UNION
        kw["flags"] = flags
    if steps > 1:
        kw["steps"] = steps
    return kw


def gpu_search(idx, q, K, L, visited="hash", allow_cap=False, **kw):
    s = song()
    p = s.Params(K=K, queue_len=L, visited=visited, **kw)
    qt = torch.as_tensor(q, device="cuda")
    ids, d, c = idx.search(qt, params=p, counters=True)
    torch.cuda.synchronize()
    try:
        idx.last_status()
    except s.SongError as e:
        if not (allow_cap and e.code == -5):
            raise
    return ids.cpu().numpy(), d.cpu().numpy(), c.cpu().numpy()


def bloom_bits_for(L, log2=0, visited="bloom"):
    """The oracle's filter size for a GPU run: Bloom bits or Cuckoo buckets."""
    if log2:
        return 1 << log2
    return oracle.default_cuckoo_buckets(L) if visited == "cuckoo" else oracle.default_bloom_bits(L)


def assert_exact(g, o):
    gi, gd, gc = g
    oi, od, oc = o[:3]
    np.testing.assert_array_equal(gi, oi)
    np.testing.assert_array_equal(gd, od)
    np.testing.assert_array_equal(gc.astype(np.int64), oc)


def assert_close(g, o, truth=None, id_frac=0.995, scale=1.0):
    gi, gd, _ = g
    oi, od = o[0], o[1]
    same = (gi == oi).all(1).mean()
    assert same >= id_frac, f"only {same:.4f} of queries have identical top-K ids"
    ok = gi == oi
    np.testing.assert_allclose(gd[ok], od[ok], rtol=1e-5, atol=1e-5 * scale)
    if truth is not None:
        assert abs(oracle.recall(gi, truth) - oracle.recall(oi, truth)) <= 0.002


# ---------------------------------------------------------------- toy / P1-P2
@pytest.mark.parametrize("visited", ALL_VISITED)
def test_fig1_toy_on_gpu(visited):
    data, adj, _, result = pins.load_toy()
    s = song()
    idx = s.SongIndex(data, adj)
    ids, d, c = gpu_search(idx, np.zeros((1, 1), np.float32), 3, 3, visited)
    assert [int(x) + 1 for x in ids[0]] == result
    o = oracle.search(data, adj, np.zeros((1, 1), np.float32), 3, 3,
                      **oracle_kw(visited, 3, idx=idx))
    assert_exact((ids, d, c), o)
    if visited == "hash":
        # the paper's literal structures (separate q and topk) with its literal
        # (eager) deletion: Fig. 4(c), 12 distances, 4 expansions
        ids, d, c = gpu_search(idx, np.zeros((1, 1), np.float32), 3, 3, visited, visited_cap=-1,
                               queue_kind="separate")
        assert [int(x) + 1 for x in ids[0]] == result
        assert c[0].tolist() == [12, 4]
        # lazy deletion with the default capacity (R14): no vertex recomputed here
        assert gpu_search(idx, np.zeros((1, 1), np.float32), 3, 3,
                          queue_kind="separate")[2][0].tolist() == [10, 4]
        # the bounded union (R17, the default): the same ids and pops; its eager
        # deletion differs from Fig. 4(c)'s (a key leaves W, not q or topk)
        for cap in (0, -1):
            g = gpu_search(idx, np.zeros((1, 1), np.float32), 3, 3, visited, visited_cap=cap,
                           queue_kind="union")
            assert [int(x) + 1 for x in g[0][0]] == result and g[2][0][1] == 4
            o = oracle.search(data, adj, np.zeros((1, 1), np.float32), 3, 3,
                              **oracle_kw(visited, 3, visited_cap=cap, queue_kind="union", idx=idx))
            assert_exact(g, o)


# ----------------------------------------------------------------- tiny config
@pytest.fixture(scope="module")
def tiny():
    cfg = CONFIGS["tiny"]
    x, q = make_data(cfg)
    adj = build_graph(x, degree=cfg.degree, row_block=2048, col_block=16384).numpy()
    xn, qn = x.numpy(), q.numpy()
    truth, _ = oracle.bruteforce(xn, qn, cfg.K, nthreads=8)
    return cfg, xn, qn, adj, truth


@pytest.mark.parametrize("L", [10, 64, 257])
@pytest.mark.parametrize("visited", ALL_VISITED)
def test_tiny_parity(tiny, L, visited):
    cfg, x, q, adj, truth = tiny
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q, cfg.K, L, visited)
    o = oracle.search(x, adj, q, cfg.K, L, **oracle_kw(visited, L, idx=idx))
    assert_close(g, o, truth, scale=float(np.abs(o[1]).max()))


# -------------------------------------------- integer data: bit-exact (P8)
@pytest.fixture(scope="module")
def sift100k():
    cfg = CONFIGS["sift1m"]
    x, q = make_data(cfg, device="cuda", n=100_000, nq=500)
    adj = build_graph(x, degree=32)
    return cfg, x, q, adj


@pytest.mark.parametrize("L,visited,warps", [(10, "hash", 4), (16, "hash", 1), (64, "hash", 4),
                                            (200, "hash", 3), (64, "bloom", 4),
                                            (1024, "hash", 2), (48, "hashtable", 4),
                                            (48, "hashtable-sel", 2), (48, "cuckoo", 4),
                                            (300, "cuckoo", 2), (300, "hashtable-sel", 4)])
def test_sift_integer_bit_exact(sift100k, L, visited, warps):
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q.cpu().numpy(), cfg.K, L, visited, warps_per_block=warps)
    o = oracle.search(x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy(), cfg.K, L,
                      **oracle_kw(visited, L, idx=idx),
                      nthreads=8)
    assert_exact(g, o)


def test_sift_small_cuckoo_filter_exact(sift100k):
    """A 16/64-bucket Cuckoo filter overflows constantly: kicks, drops,
    fingerprint collisions and the false negatives they cause (re-admitted
    vertices) must follow the oracle's order exactly.  A lossy filter
    can make the search revisit forever, so both sides cap expansions."""
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    for L in (24, 160):
        for tl in (4, 6):
            g = gpu_search(idx, q.cpu().numpy(), cfg.K, L, "cuckoo", allow_cap=True,
                           table_log2=tl, max_iters=3000)
            o = oracle.search(x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy(), cfg.K, L,
                              flags=oracle.OPTIMIZED_CUCKOO, bloom_bits=1 << tl, nthreads=8,
                              max_iters=3000)
            assert_exact(g, o)


def test_global_table_full_is_reported(sift100k):
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    with pytest.raises(s.SongError, match="EUNSUPPORTED"):
        gpu_search(idx, q.cpu().numpy()[:32], cfg.K, 64, "hashtable", table_log2=6)


def test_sift_small_bloom_filter_exact(sift100k):
    """A deliberately small Bloom filter (2^9 bits) saturates: false positives
    change the search, and the GPU must follow the oracle's spec bit by bit."""
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q.cpu().numpy(), cfg.K, 48, "bloom", bloom_log2_bits=9)
    o = oracle.search(x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy(), cfg.K, 48,
                      flags=oracle.OPTIMIZED_BLOOM, bloom_bits=1 << 9, nthreads=8)
    assert_exact(g, o)


def test_host_and_device_entry_points_agree(sift100k):
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)  # device create
    idx2 = s.SongIndex(x.cpu().numpy(), adj.cpu().numpy())  # host create
    qi, qd = idx2.search_host(q.cpu().numpy(), cfg.K, 64)
    g = gpu_search(idx, q.cpu().numpy(), cfg.K, 64)
    np.testing.assert_array_equal(qi, g[0])
    np.testing.assert_array_equal(qd, g[1])


@pytest.mark.parametrize("L,visited,nbatch", [(64, "hash", 5), (16, "hash", 1), (48, "hashtable", 4),
                                             (1024, "hash", 3), (48, "cuckoo", 2)])
def test_pipelined_batches_match_single_searches(sift100k, L, visited, nbatch):
    """song_search_pipelined (two lanes in flight, copy streams, the next
    batch's kernel in the previous one's tail) returns, batch by batch, what
    song_search_ex returns for that batch alone — and the oracle's answer."""
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    qn = q.cpu().numpy()
    nq = qn.shape[0] // nbatch
    qb = np.ascontiguousarray(qn[:nq * nbatch].reshape(nbatch, nq, -1))
    p = s.Params(K=cfg.K, queue_len=L, visited=visited)
    ids, dists = idx.search_pipelined(qb, p)
    for b in range(nbatch):
        g = gpu_search(idx, qb[b], cfg.K, L, visited)
        np.testing.assert_array_equal(ids[b], g[0])
        np.testing.assert_array_equal(dists[b], g[1])
    o = oracle.search(x.cpu().numpy(), adj.cpu().numpy(), qb.reshape(nq * nbatch, -1), cfg.K, L,
                      nthreads=8, **oracle_kw(visited, L, idx=idx))
    np.testing.assert_array_equal(ids.reshape(nq * nbatch, -1), o[0])
    np.testing.assert_array_equal(dists.reshape(nq * nbatch, -1), o[1])
    # the call is repeatable (lanes and events are reused) and ordered after
    # a device search enqueued just before it on torch's stream
    idx.search(q, params=p)
    ids2, dists2 = idx.search_pipelined(qb, p)
    np.testing.assert_array_equal(ids2, ids)


def test_pipelined_large_batches_overlap(sift100k):
    """Batches larger than the resident grid (outlier-first order, tails
    overlapping the next batch's kernel) on pinned host buffers."""
    cfg, x, _, adj = sift100k
    s = song()
    _, qbig = make_data(cfg, device="cpu", n=1000, nq=12_000)
    qb = torch.empty((3, 4000, cfg.dim), dtype=torch.float32, pin_memory=True)
    qb.copy_(qbig.reshape(3, 4000, -1))
    ih = torch.empty((3, 4000, cfg.K), dtype=torch.int32, pin_memory=True)
    dh = torch.empty((3, 4000, cfg.K), dtype=torch.float32, pin_memory=True)
    idx = s.SongIndex(x, adj)
    p = s.Params(K=cfg.K, queue_len=32)
    idx.search_pipelined_into(qb, p, ih, dh)
    for b in range(3):
        g = gpu_search(idx, qb[b].numpy(), cfg.K, 32)
        np.testing.assert_array_equal(ih[b].numpy(), g[0])
        np.testing.assert_array_equal(dh[b].numpy(), g[1])


def test_search_host_large_batch(sift100k):
    """song_search on a batch of several resident grids' worth (outlier-first
    order, a ragged tail) and then a small call: the device search's results."""
    cfg, x, _, adj = sift100k
    s = song()
    _, qbig = make_data(cfg, device="cpu", n=1000, nq=12_001)  # ragged last chunk
    idx = s.SongIndex(x, adj)
    hi, hd = idx.search_host(qbig.numpy(), cfg.K, 24)
    g = gpu_search(idx, qbig.numpy(), cfg.K, 24)
    np.testing.assert_array_equal(hi, g[0])
    np.testing.assert_array_equal(hd, g[1])
    hi2, _ = idx.search_host(qbig.numpy()[:100], cfg.K, 24)  # then a small unchunked call
    np.testing.assert_array_equal(hi2, g[0][:100])


def test_pipelined_argument_errors(sift100k):
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    qb = np.zeros((2, 4, cfg.dim), np.float32)
    with pytest.raises(s.SongError, match="EINVAL"):
        idx.search_pipelined(qb, s.Params(K=10, queue_len=5))
    qb[1, 2, 3] = np.nan  # a non-finite query in the second batch: sticky status
    with pytest.raises(s.SongError, match="EINVAL"):
        idx.search_pipelined(qb, s.Params(K=10, queue_len=16))


# ------------------------------------------------ other metrics / dimensions
@pytest.mark.parametrize("name,n", [("glove200", 30_000), ("nytimes256", 30_000),
                                    ("gist1m", 20_000)])
def test_metric_and_dim_parity(name, n):
    cfg = CONFIGS[name]
    x, q = make_data(cfg, device="cuda", n=n, nq=200)
    adj = build_graph(x, degree=cfg.degree, metric=cfg.metric)
    s = song()
    idx = s.SongIndex(x, adj, metric=cfg.metric)
    xn, qn, an = x.cpu().numpy(), q.cpu().numpy(), adj.cpu().numpy()
    m = oracle.METRICS[cfg.metric]
    truth, _ = oracle.bruteforce(xn, qn, cfg.K, metric=m, nthreads=8)
    for L in (32, 128):
        g = gpu_search(idx, qn, cfg.K, L)
        o = oracle.search(xn, an, qn, cfg.K, L, metric=m, nthreads=8)
        assert_close(g, o, truth, id_frac=0.995,
                     scale=float(np.abs(o[1]).max()))


# ------------------------------------------------------------------- edges
def small_random(n=3000, dim=30, deg=12, seed=0, integer=True):
    rng = np.random.default_rng(seed)
    x = rng.integers(0, 20, (n, dim)).astype(np.float32) if integer else \
        rng.standard_normal((n, dim)).astype(np.float32)
    adj = rng.integers(-1, n, (n, deg)).astype(np.int32)
    adj[:, 0] = (np.arange(n) + 1) % n
    adj[:, 3] = adj[:, 2]  # repeated ids inside a row
    q = rng.integers(0, 20, (64, dim)).astype(np.float32) if integer else \
        rng.standard_normal((64, dim)).astype(np.float32)
    return x, adj, q


@pytest.mark.parametrize("dim", [1, 3, 30, 130, 257])
@pytest.mark.parametrize("L,K", [(1, 1), (7, 7), (33, 10), (100, 100), (150, 20)])
def test_edges_exact(dim, L, K):
    """ragged dims (row padding), degree < 32 with -1 padding and repeats,
    L = K = 1 (greedy), K = L, queue sizes that are not multiples of 32."""
    x, adj, q = small_random(dim=dim)
    s = song()
    idx = s.SongIndex(x, adj)
    for visited in ALL_VISITED:
        g = gpu_search(idx, q, K, L, visited)
        o = oracle.search(x, adj, q, K, L, **oracle_kw(visited, L, idx=idx))
        assert_exact(g, o)
    for qk in ("union", "separate"):  # every queue kind at every L (R17 / §IV-C)
        for cap in (0, -1):
            g = gpu_search(idx, q, K, L, "hash", queue_kind=qk, visited_cap=cap)
            o = oracle.search(x, adj, q, K, L, **oracle_kw("hash", L, visited_cap=cap, queue_kind=qk, idx=idx))
            assert_exact(g, o)


@pytest.mark.parametrize("L", [129, 200, 640, 1280])
@pytest.mark.parametrize("cap", [0, -1, "min"])
def test_union_queue_bit_exact(sift100k, L, cap):
    """Reading R17 (the default above 128): ids, distances and counters
    bit-exact against the oracle's bounded-union mode, every deletion
    schedule; results equal the separate q / topk structures (§IV-C)."""
    cfg, x, q, adj = sift100k
    cap = L + 32 if cap == "min" else cap
    s = song()
    idx = s.SongIndex(x, adj)
    xn, an, qn = x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy()[:200]
    g = gpu_search(idx, qn, cfg.K, L, "hash", visited_cap=cap)
    o = oracle.search(xn, an, qn, cfg.K, L, nthreads=8, **oracle_kw("hash", L, visited_cap=cap, idx=idx))
    assert o is not None and s.plan(s.Params(K=1, queue_len=L), 128).queue_kind == 2
    assert_exact(g, o)
    sep = gpu_search(idx, qn, cfg.K, L, "hash", queue_kind="separate")
    np.testing.assert_array_equal(g[0], sep[0])
    np.testing.assert_array_equal(g[1], sep[1])
    np.testing.assert_array_equal(g[2][:, 1], sep[2][:, 1])  # the same popped sequence


@pytest.mark.parametrize("L", [10, 16, 48, 100, 128])
@pytest.mark.parametrize("cap", [0, -1, "min"])
def test_register_union_bit_exact(sift100k, L, cap):
    """Reading R17 with W in registers (queue_kind "union" at queue_len <=
    128): bit-exact against the oracle's bounded-union mode, every deletion
    schedule, and the same results and pops as the separate register q /
    topk of §IV-C."""
    cfg, x, q, adj = sift100k
    cap = L + 32 if cap == "min" else cap
    s = song()
    idx = s.SongIndex(x, adj)
    K = min(cfg.K, L)
    xn, an, qn = x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy()
    pl = idx.plan(s.Params(K=K, queue_len=L, queue_kind="union"))
    assert pl.queue_kind == 2 and pl.queue_regs == (1 if L <= 32 else 2 if L <= 64 else 4)
    g = gpu_search(idx, qn, K, L, "hash", visited_cap=cap, queue_kind="union")
    o = oracle.search(xn, an, qn, K, L, nthreads=8,
                      **oracle_kw("hash", L, visited_cap=cap, queue_kind="union", idx=idx))
    assert_exact(g, o)
    sep = gpu_search(idx, qn, K, L, "hash", queue_kind="separate")
    np.testing.assert_array_equal(g[0], sep[0])
    np.testing.assert_array_equal(g[1], sep[1])
    np.testing.assert_array_equal(g[2][:, 1], sep[2][:, 1])  # the same popped sequence


def test_entry_offset_and_unreachable_padding():
    x, adj, q = small_random(n=500, dim=8)
    adj2 = adj.copy()
    adj2[:] = -1
    adj2[5, :3] = [6, 7, 8]  # only 4 vertices reachable from entry 5
    s = song()
    idx = s.SongIndex(x, adj2)
    g = gpu_search(idx, q, 10, 16, entry=5, id_offset=1000)
    assert (g[0][:, :4] >= 1000).all() and (g[0][:, 4:] == -1).all()
    assert np.isinf(g[1][:, 4:]).all()
    o = oracle.search(x, adj2, q, 10, 16, entry=5)
    np.testing.assert_array_equal(np.where(g[0] >= 0, g[0] - 1000, -1), o[0])


def test_large_queue_len_max():
    x, adj, q = small_random(n=5000, dim=16, deg=32)
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q[:16], 100, 2048)
    o = oracle.search(x, adj, q[:16], 100, 2048, **oracle_kw("hash", 2048, idx=idx))
    assert_exact(g, o)
    g = gpu_search(idx, q[:16], 100, 2048, visited_cap=-1)  # eager deletion
    o = oracle.search(x, adj, q[:16], 100, 2048, **oracle_kw("hash", 2048, visited_cap=-1, idx=idx))
    assert_exact(g, o)
    for qk in ("separate", "union"):  # both shared-memory queue kinds at the maximum
        g = gpu_search(idx, q[:16], 100, 2048, queue_kind=qk)
        o = oracle.search(x, adj, q[:16], 100, 2048, **oracle_kw("hash", 2048, queue_kind=qk, idx=idx))
        assert_exact(g, o)


def test_errors():
    s = song()
    x, adj, q = small_random(n=100, dim=4)
    bad = adj.copy()
    bad[3, 1] = 100
    with pytest.raises(s.SongError, match="EINVAL"):
        s.SongIndex(x, bad)
    with pytest.raises(s.SongError, match="EINVAL"):
        s.SongIndex(torch.as_tensor(x, device="cuda"), torch.as_tensor(bad, device="cuda"))
    xn = x.copy()
    xn[2, 2] = np.nan
    with pytest.raises(s.SongError, match="EINVAL"):
        s.SongIndex(xn, adj)
    idx = s.SongIndex(x, adj)
    with pytest.raises(s.SongError, match="EINVAL"):
        idx.search_host(q, 10, 5)  # queue_len < K
    with pytest.raises(s.SongError, match="EUNSUPPORTED"):
        idx.search_host(q, 10, 4096)
    qb = q.copy()
    qb[1, 0] = np.inf
    with pytest.raises(s.SongError, match="EINVAL"):
        idx.search_host(qb, 10, 16)
    with pytest.raises(s.SongError, match="EITERCAP"):
        gpu_search(idx, q, 10, 64, max_iters=2)


# ----------------------------------------------------------------- merge
def test_merge_topk_matches_plain_merge():
    rng = np.random.default_rng(0)
    G, nq, kin, K = 4, 300, 20, 10
    ids = np.full((G, nq, kin), -1, np.int32)
    dists = np.full((G, nq, kin), np.inf, np.float32)
    for g in range(G):
        for r in range(nq):
            m = rng.integers(0, kin + 1)
            d = np.sort(rng.integers(0, 50, m).astype(np.float32))
            i = rng.choice(1000, m, replace=False) + g * 1000
            order = np.lexsort((i, d))
            ids[g, r, :m] = i[order]
            dists[g, r, :m] = d[order]
    s = song()
    oi, od = s.merge_topk(torch.as_tensor(ids, device="cuda"), torch.as_tensor(dists, device="cuda"), K)
    ei, ed = oracle.merge_shards(list(ids), list(dists), K)
    np.testing.assert_array_equal(oi.cpu().numpy(), ei)
    np.testing.assert_array_equal(od.cpu().numpy(), ed)


def test_dataset_sharding_emulated_on_one_gpu(sift100k):
    """P:471 on one GPU: G shards searched one after another with global ids
    (id_offset), merged by song_merge_topk; bit-exact vs the oracle per shard +
    the plain merge (SURVEY §4 single-GPU emulation)."""
    from paper_conf_icde_zhaotl20_b200 import sharded
    cfg, x, q, adj = sift100k
    s = song()
    G, K, L = 3, 10, 40
    gi, gd, per_i, per_d = [], [], [], []
    for lo, hi in sharded.shard_ranges(x.shape[0], G):
        xs = x[lo:hi].contiguous()
        a = build_graph(xs, degree=32)
        idx = s.SongIndex(xs, a)
        i, d = idx.search(q, params=s.Params(K=K, queue_len=L, id_offset=lo))
        gi.append(i)
        gd.append(d)
        oi, od, _, _ = oracle.search(xs.cpu().numpy(), a.cpu().numpy(), q.cpu().numpy(), K, L,
                                     nthreads=8)
        per_i.append(np.where(oi >= 0, oi + lo, -1))
        per_d.append(od)
    mi, md = s.merge_topk(torch.stack(gi), torch.stack(gd), K)
    ei, ed = oracle.merge_shards(per_i, per_d, K)
    np.testing.assert_array_equal(mi.cpu().numpy(), ei)
    np.testing.assert_array_equal(md.cpu().numpy(), ed)
    # the fused gather + merge kernel reading the G shards' buffers through a
    # pointer table (on one GPU the "peers" are local buffers; no pads)
    ptr = lambda ts: torch.tensor([t.data_ptr() for t in ts], dtype=torch.int64, device="cuda")  # noqa: E731
    fi, fd = s.merge_topk_peers(ptr(gi), ptr(gd), q.shape[0], K, K)
    np.testing.assert_array_equal(fi.cpu().numpy(), ei)
    np.testing.assert_array_equal(fd.cpu().numpy(), ed)
    # ... and with signal pads: one pad per "rank", every rank's merge signals
    # all pads first (here all G merges run on one GPU, one after another, so
    # rank g waits only on the pads already set: run them in reverse order of
    # need by pre-setting the other ranks' slots)
    pads = [torch.zeros(G, dtype=torch.int32, device="cuda") for _ in range(G)]
    for g in range(G):
        for h in range(G):
            pads[g][h] = 7  # every peer already signalled epoch 7
    for g in range(G):
        pi, pd = s.merge_topk_peers(ptr(gi), ptr(gd), q.shape[0], K, K, sig_ptrs=ptr(pads),
                                    rank=g, epoch=7)
        np.testing.assert_array_equal(pi.cpu().numpy(), ei)
        np.testing.assert_array_equal(pd.cpu().numpy(), ed)
    torch.cuda.synchronize()
    assert all(int(p[g]) == 7 for g, p in enumerate(pads))


def test_fused_peer_merge_over_symmetric_memory(sift100k, tmp_path):
    """The product path of dataset sharding (ShardedIndex.search, NCCL): the
    search writes into symmetric-memory buffers and song_merge_topk_peers
    signals and merges — on a one-rank NCCL group here (the driver's boxes
    have one GPU), bit-exact against the oracle's per-shard search + merge."""
    import torch.distributed as dist
    from paper_conf_icde_zhaotl20_b200 import sharded
    cfg, x, q, adj = sift100k
    s = song()
    store = dist.FileStore(str(tmp_path / "store"), 1)
    dist.init_process_group("nccl", store=store, rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        K, L = 10, 40
        si = sharded.ShardedIndex(x, adj, id_offset=0)
        for _ in range(2):  # the second call reuses the buffers (epoch 2)
            fi, fd = si.search(q, q.shape[0], K, L, fused=True)
            torch.cuda.synchronize()
        assert si._merger.epoch == 2
        oi, od, _, _ = oracle.search(x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy(), K, L,
                                     nthreads=8, **oracle_kw("hash", L, idx=si.index))
        ei, ed = oracle.merge_shards([oi], [od], K)
        np.testing.assert_array_equal(fi.cpu().numpy(), ei)
        np.testing.assert_array_equal(fd.cpu().numpy(), ed)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("L", [10, 48, 64, 128, 200])
@pytest.mark.parametrize("cap", [-1, 0, "min"])
def test_deletion_schedules_exact(sift100k, L, cap):
    """Reading R14: eager (-1), default lazy (0) and the smallest lazy capacity
    2L + 32 — identical results, each schedule's own counters bit-exact."""
    cfg, x, q, adj = sift100k
    cap = 2 * L + 32 if cap == "min" else cap
    s = song()
    idx = s.SongIndex(x, adj)
    xn, an, qn = x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy()
    g = gpu_search(idx, qn, cfg.K, L, "hash", visited_cap=cap)
    o = oracle.search(xn, an, qn, cfg.K, L, nthreads=8, **oracle_kw("hash", L, visited_cap=cap, idx=idx))
    assert_exact(g, o)
    eager = oracle.search(xn, an, qn, cfg.K, L, nthreads=8, **oracle_kw("hash", L, visited_cap=-1, idx=idx))
    np.testing.assert_array_equal(g[0], eager[0])  # the schedule never changes results
    np.testing.assert_array_equal(g[1], eager[1])
    if cap != -1:
        assert g[2][:, 0].sum() <= eager[2][:, 0].sum()  # ... only the recomputations


@pytest.mark.slow
def test_sift1m_full_size_sampled_parity():
    """BASELINE configs[1] at full size (1M x 128, degree 32, 10,000 queries) in
    bench.py's launch configuration (default launch shape, queue_len 48 = the
    recall@10 >= 0.95 operating point): the oracle recomputes a sample of 300
    queries one by one; ids, distances and counters must be bit-exact."""
    cfg = CONFIGS["sift1m"]
    x, q = make_data(cfg, device="cuda")
    adj = build_graph(x, degree=cfg.degree)
    s = song()
    idx = s.SongIndex(x, adj)
    ids, d, c = idx.search(q, params=s.Params(K=cfg.K, queue_len=48), counters=True)
    torch.cuda.synchronize()
    idx.last_status()
    rng = np.random.default_rng(0)
    pick = np.sort(rng.choice(cfg.nq, 300, replace=False))
    xn, an = x.cpu().numpy(), adj.cpu().numpy()
    o = oracle.search(xn, an, q.cpu().numpy()[pick], cfg.K, 48, nthreads=8,
                      **oracle_kw("hash", 48, idx=idx))
    assert_exact((ids.cpu().numpy()[pick], d.cpu().numpy()[pick], c.cpu().numpy()[pick]), o)
    # properties that hold for every query at any size: sorted, unique, valid ids
    ii, dd = ids.cpu().numpy(), d.cpu().numpy()
    assert (np.diff(dd, axis=1) >= 0).all()
    assert ((ii >= 0) & (ii < cfg.n)).all()
    assert all(len(set(r)) == cfg.K for r in ii)


@pytest.mark.parametrize("visited,steps,L", [("bloom", 1, 48), ("cuckoo", 1, 48),
                                             ("hashtable-sel", 1, 48), ("hash", 2, 48),
                                             ("hash", 1, 600)])
def test_schedule_other_paths(sift100k, visited, steps, L):
    """Outlier-first order on the other kernel variants (Bloom / Cuckoo / global
    hash, multi-step probing, shared-memory queues): identical to batch order."""
    cfg, x, q, adj = sift100k
    s = song()
    idx = s.SongIndex(x, adj)
    qq = q.repeat(8, 1).contiguous()  # 4000 queries > 148 x 24 resident warps
    res = []
    for sched in ("batch", "outlier_first"):
        ids, d, c = idx.search(qq, params=s.Params(K=cfg.K, queue_len=L, visited=visited,
                                                   steps=steps, schedule=sched), counters=True)
        torch.cuda.synchronize()
        idx.last_status()
        res.append((ids.cpu().numpy(), d.cpu().numpy(), c.cpu().numpy()))
    for a, b in zip(*res):
        np.testing.assert_array_equal(a, b)
    idx.close()


@pytest.mark.parametrize("name,L", [("sift1m", 48), ("glove200", 64), ("nytimes256", 64)])
def test_schedule_never_changes_results(name, L):
    """The outlier-first ticket order (song_search_params.schedule) only moves
    queries between warps: ids, distances and counters equal the batch order's
    for every query, and the oracle's on a sample (integer data: bit-exact)."""
    s = song()
    cfg = CONFIGS[name]
    x, q = make_data(cfg, device="cuda", n=50_000, nq=6000)  # > 148 x 24 resident warps
    adj = s.build_graph(x, cfg.degree, cfg.metric)
    idx = s.SongIndex(x, adj, metric=cfg.metric)
    res = {}
    for sched in ("batch", "outlier_first", "auto"):
        ids, d, c = idx.search(q, params=s.Params(K=cfg.K, queue_len=L, schedule=sched),
                               counters=True)
        torch.cuda.synchronize()
        idx.last_status()
        res[sched] = (ids.cpu().numpy(), d.cpu().numpy(), c.cpu().numpy())
    for sched in ("outlier_first", "auto"):
        for a, b in zip(res["batch"], res[sched]):
            np.testing.assert_array_equal(a, b)
    pick = np.arange(0, 6000, 40)
    o = oracle.search(x.cpu().numpy(), adj.cpu().numpy(), q.cpu().numpy()[pick], cfg.K, L,
                      metric=oracle.METRICS[cfg.metric], nthreads=8, **oracle_kw("hash", L, idx=idx))
    g = tuple(r[pick] for r in res["outlier_first"])
    if cfg.kind == "sift":
        assert_exact(g, o)
    else:
        assert_close(g, o, scale=float(np.abs(o[1]).max()), id_frac=0.995)
    p = s.Params(K=cfg.K, queue_len=L).to_c()
    p.schedule = 7
    out = torch.empty((1, cfg.K), dtype=torch.int32, device="cuda")
    rc = s.lib().song_search_ex(idx._h, ctypes.byref(p), ctypes.c_void_p(q.data_ptr()), 1,
                                ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                None, None)
    assert rc == -1 and b"schedule" in s.lib().song_last_error()
    idx.close()


@pytest.mark.parametrize("dim", [1020, 1024])  # SONG_MAX_DIM: 8 chunks per lane, ragged last one
def test_max_dim_exact(dim):
    x, adj, q = small_random(n=2000, dim=dim)
    s = song()
    idx = s.SongIndex(x, adj)
    for visited in ("hash", "bloom"):
        g = gpu_search(idx, q, 10, 40, visited)
        o = oracle.search(x, adj, q, 10, 40, **oracle_kw(visited, 40, idx=idx))
        assert_exact(g, o)
    idx.close()


def test_single_vertex_and_isolated_entry():
    """n = 1 (the entry is the only vertex), and an entry whose row is all
    padding: one distance, one expansion, the rest of the output padded."""
    s = song()
    x = np.array([[3.0, 4.0]], np.float32)
    idx = s.SongIndex(x, np.full((1, 4), -1, np.int32))
    g = gpu_search(idx, np.zeros((2, 2), np.float32), 3, 4)
    o = oracle.search(x, np.full((1, 4), -1, np.int32), np.zeros((2, 2), np.float32), 3, 4,
                      **oracle_kw("hash", 4, idx=idx))
    assert_exact(g, o)
    assert (g[0][:, 0] == 0).all() and (g[0][:, 1:] == -1).all()
    assert (g[1][:, 0] == 25.0).all() and np.isinf(g[1][:, 1:]).all()
    assert (g[2] == [[1, 1]]).all()
    idx.close()


def test_stage_cycles_only_in_instrumented_builds():
    """song_stage_cycles: the product library is built without
    SONG_STAGE_TIMING and says so (SONG_EUNSUPPORTED, zeroed output)."""
    x, adj, q = small_random(n=300, dim=8)
    s = song()
    idx = s.SongIndex(x, adj)
    gpu_search(idx, q, 10, 16)
    with pytest.raises(s.SongError) as e:
        idx.stage_cycles()
    assert e.value.code == -4


def test_search_plan_matches_the_launch():
    """The plan (song_search_plan_get, host-only) is what the search runs: the
    lazy capacity it reports reproduces the GPU's counters in the oracle for a
    narrow (NCH 1) and a wide (NCH 2) row, where the table sizes differ."""
    s = song()
    for dim in (16, 200):
        x, adj, q = small_random(n=2000, dim=dim, deg=16)
        idx = s.SongIndex(x, adj)
        for L in (32, 64, 100, 200):
            pl = idx.plan(s.Params(K=10, queue_len=L))
            assert pl.visited_cap > 0
            g = gpu_search(idx, q, 10, L)
            flags = oracle.OPTIMIZED_LAZY | (oracle.UNION if pl.queue_kind == 2 else 0)
            o = oracle.search(x, adj, q, 10, L, flags=flags, lazy_cap=pl.visited_cap)
            assert_exact(g, o)
