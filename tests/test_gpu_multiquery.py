"""GPU parity of Fig. 8's multi-query packing (§V):
song_search_params.queries_per_warp = 1, 2 or 4 runs that many queries per
warp, each on its own team of 32 / G lanes.  Its schedule is the paper's
literal one (separate q / topk, selected insertion, eager deletion), so it
is compared with the oracle's OPTIMIZED mode: bit-exact ids, distances and
counters on integer-valued data, the north-star bars on float data, and
the same ids / distances / pops as the production kernel."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from workloads.graph import build_graph  # noqa: E402
from workloads.synth import CONFIGS, make_data  # noqa: E402

import test_oracle_pins as pins  # noqa: E402
from test_gpu_parity import assert_close, assert_exact, gpu_search, small_random, song  # noqa: E402

GS = [1, 2, 4]


@pytest.mark.parametrize("G", GS)
def test_fig1_toy_packed(G):
    """Fig. 1's toy under the paper's literal schedule: ids 8, 2, 7 and
    Fig. 4(c)'s 12 distances / 4 expansions with any packing."""
    data, adj, _, result = pins.load_toy()
    s = song()
    idx = s.SongIndex(data, adj)
    q = np.zeros((3, 1), np.float32)  # three identical queries share warps when G > 1
    g = gpu_search(idx, q, 3, 3, visited_cap=-1, queries_per_warp=G)
    for r in range(3):
        assert [int(x) + 1 for x in g[0][r]] == result
        assert g[2][r].tolist() == [12, 4]
    o = oracle.search(data, adj, q, 3, 3, flags=oracle.OPTIMIZED)
    assert_exact(g, o)


@pytest.fixture(scope="module")
def sift50k():
    cfg = CONFIGS["sift1m"]
    x, q = make_data(cfg, device="cuda", n=50_000, nq=301)  # 301: a ragged last warp
    adj = build_graph(x, degree=32)
    return cfg, x.cpu().numpy(), q.cpu().numpy(), adj.cpu().numpy()


@pytest.mark.parametrize("G", GS)
@pytest.mark.parametrize("L", [10, 16, 33, 64, 100, 128])
def test_sift_packed_bit_exact(sift50k, G, L):
    cfg, x, q, adj = sift50k
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q, cfg.K, L, visited_cap=-1, queries_per_warp=G)
    o = oracle.search(x, adj, q, cfg.K, L, flags=oracle.OPTIMIZED, nthreads=8)
    assert_exact(g, o)
    # the production kernel (union W, lazy deletion): same ids, distances, pops
    d = gpu_search(idx, q, cfg.K, L)
    np.testing.assert_array_equal(g[0], d[0])
    np.testing.assert_array_equal(g[1], d[1])
    np.testing.assert_array_equal(g[2][:, 1], d[2][:, 1])
    idx.close()


@pytest.mark.parametrize("G", GS)
@pytest.mark.parametrize("dim", [1, 3, 130])
@pytest.mark.parametrize("L,K", [(1, 1), (7, 7), (40, 10)])
def test_packed_edges(G, dim, L, K):
    """ragged dims, -1 padding and repeated ids in a row, greedy L = 1."""
    x, adj, q = small_random(dim=dim)
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q, K, L, visited_cap=-1, queries_per_warp=G)
    o = oracle.search(x, adj, q, K, L, flags=oracle.OPTIMIZED)
    assert_exact(g, o)
    idx.close()


@pytest.mark.parametrize("name,n", [("nytimes256", 20_000), ("glove200", 20_000)])
def test_packed_float_metrics(name, n):
    cfg = CONFIGS[name]
    x, q = make_data(cfg, device="cuda", n=n, nq=200)
    adj = build_graph(x, degree=cfg.degree, metric=cfg.metric)
    s = song()
    idx = s.SongIndex(x, adj, metric=cfg.metric)
    xn, qn, an = x.cpu().numpy(), q.cpu().numpy(), adj.cpu().numpy()
    truth, _ = oracle.bruteforce(xn, qn, cfg.K, metric=oracle.METRICS[cfg.metric], nthreads=8)
    o = oracle.search(xn, an, qn, cfg.K, 64, flags=oracle.OPTIMIZED,
                      metric=oracle.METRICS[cfg.metric], nthreads=8)
    for G in GS:
        g = gpu_search(idx, qn, cfg.K, 64, visited_cap=-1, queries_per_warp=G)
        assert_close(g, o, truth=truth, scale=float(np.abs(o[1]).max()))
    idx.close()


def test_packed_argument_errors(sift50k):
    cfg, x, q, adj = sift50k
    s = song()
    idx = s.SongIndex(x, adj)
    with pytest.raises(s.SongError, match="EINVAL"):
        gpu_search(idx, q[:4], 10, 16, visited_cap=-1, queries_per_warp=3)
    for kw in ({"visited_cap": 0}, {"visited_cap": -1, "steps": 2},
               {"visited_cap": -1, "queue_kind": "union"}, {"visited": "bloom"}):
        kw = {"queries_per_warp": 2, **kw}
        with pytest.raises(s.SongError, match="EUNSUPPORTED"):
            gpu_search(idx, q[:4], 10, 16, **kw)
    with pytest.raises(s.SongError, match="EUNSUPPORTED"):
        gpu_search(idx, q[:4], 10, 129, visited_cap=-1, queries_per_warp=2)
    plan = idx.plan(s.Params(K=10, queue_len=64, visited_cap=-1, queries_per_warp=4))
    assert plan.queue_kind == 1 and plan.visited_cap == -1  # separate q / topk, eager
    idx.close()
