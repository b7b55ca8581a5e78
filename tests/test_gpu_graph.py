"""GPU parity of the device graph builder (song_build_graph, reading R15)
against the oracle's construction: bit-exact adjacency on integer-valued data
(every distance an exact integer, ties broken by id), the hand-worked toy,
and property/agreement checks on float data and the other metrics."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from workloads.synth import CONFIGS, make_data  # noqa: E402

import test_oracle_graph as og  # noqa: E402


def song():
    from paper_conf_icde_zhaotl20_b200 import song as s
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return s


def gbuild(x, D, metric="l2"):
    adj = song().build_graph(torch.as_tensor(x, device="cuda"), D, metric)
    torch.cuda.synchronize()
    return adj.cpu().numpy()


def test_toy():
    x, want = og.load_toy()
    np.testing.assert_array_equal(gbuild(x, 2), want)


@pytest.mark.parametrize("path", ["auto", "simt", "tc"])
@pytest.mark.parametrize("n,dim,D", [(1, 4, 4), (2, 4, 4), (63, 8, 4), (64, 8, 8), (65, 12, 8),
                                     (127, 4, 16), (129, 36, 16), (300, 4, 16), (1000, 32, 32),
                                     (777, 132, 12), (2100, 64, 32)])
def test_integer_random_bit_exact(n, dim, D, path, monkeypatch):
    """ragged n (tile tails: 64-row SIMT tiles, 128-row tensor-core tiles),
    ragged dims (k tails), many exact ties; both forward-list paths (the
    tensor-core path is exact on these small integers: dim * max^2 < 2^24)."""
    if path != "auto":
        monkeypatch.setenv("SONG_GRAPH_PATH", path)
    rng = np.random.default_rng(n + dim + D)
    x = rng.integers(0, 12, (n, dim)).astype(np.float32)
    np.testing.assert_array_equal(gbuild(x, D), oracle.build_graph(x, D, nthreads=8))


@pytest.mark.parametrize("path", ["tc", "simt"])
def test_sift_shaped_bit_exact(path, monkeypatch):
    monkeypatch.setenv("SONG_GRAPH_PATH", path)
    cfg = CONFIGS["sift1m"]
    x, _ = make_data(cfg, n=6000, nq=1)
    xn = x.numpy()
    np.testing.assert_array_equal(gbuild(xn, 32), oracle.build_graph(xn, 32, nthreads=8))


def test_odd_dims_take_the_simt_path():
    """dim % 4 != 0 (no 16 B TMA rows) and non-tf32 values use fp32 FFMA tiles."""
    rng = np.random.default_rng(1)
    x = rng.integers(0, 9, (500, 7)).astype(np.float32)
    np.testing.assert_array_equal(gbuild(x, 8), oracle.build_graph(x, 8))


@pytest.mark.parametrize("metric", ["l2", "ip", "cosine"])
def test_float_data_agrees(metric):
    """fp32 GPU arithmetic vs the oracle's fp64: rows agree except at near-ties."""
    rng = np.random.default_rng(3)
    x = rng.standard_normal((2000, 24)).astype(np.float32)
    g = gbuild(x, 16, metric)
    o = oracle.build_graph(x, 16, metric=oracle.METRICS[metric], nthreads=8)
    same_sets = np.mean([set(a) == set(b) for a, b in zip(g, o)])
    assert same_sets >= 0.99, same_sets
    assert ((g >= -1) & (g < len(x))).all()


def test_search_quality_on_the_built_graph():
    """The graph the builder makes is searchable: recall@10 at L = 64 on a
    SIFT-shaped 50K set matches the tooling graph's."""
    from workloads.graph import build_graph as tool_build
    cfg = CONFIGS["sift1m"]
    x, q = make_data(cfg, device="cuda", n=50_000, nq=500)
    s = song()
    truth, _ = oracle.bruteforce(x.cpu().numpy(), q.cpu().numpy(), 10, nthreads=8)
    recs = []
    for adj in (s.build_graph(x, 32), tool_build(x, degree=32)):
        idx = s.SongIndex(x, adj)
        ids, _ = idx.search(q, params=s.Params(K=10, queue_len=64))
        torch.cuda.synchronize()
        recs.append(oracle.recall(ids.cpu().numpy(), truth))
        idx.close()
    assert recs[0] >= 0.95 and abs(recs[0] - recs[1]) < 0.01, recs


def test_errors():
    s = song()
    x = torch.zeros((10, 4), device="cuda")
    for D, code in ((0, -1), (33, -4)):
        with pytest.raises(s.SongError) as e:
            s.build_graph(x, D)
        assert e.value.code == code


# ------------------------------------------- batched insertion (reading R16)
def gbuild_batched(x, D, metric="l2", **kw):
    adj = song().build_graph_batched(torch.as_tensor(x, device="cuda"), D, metric, **kw)
    torch.cuda.synchronize()
    return adj.cpu().numpy()


@pytest.mark.parametrize("n,dim,D,prefix,L,shift", [
    (600, 8, 6, 100, 600, 1),      # exhaustive searches (the pinned special case)
    (3000, 30, 12, 200, 32, 1),    # dim % 4 != 0: the padded search view
    (5000, 16, 16, 500, 48, 0),    # doubling batches
    (4097, 64, 32, 1000, 64, 2),   # ragged last batch
])
def test_batched_integer_bit_exact(n, dim, D, prefix, L, shift):
    x = og._int_data(n, dim, n)
    want = oracle.build_graph_batched(x, D, prefix=prefix, queue_len=L, batch_shift=shift,
                                      nthreads=8)
    np.testing.assert_array_equal(gbuild_batched(x, D, prefix=prefix, queue_len=L,
                                                 batch_shift=shift), want)


def test_batched_sift_shaped_bit_exact():
    cfg = CONFIGS["sift1m"]
    x, _ = make_data(cfg, device="cuda", n=20_000, nq=1)
    got = gbuild_batched(x, 32, prefix=2000, queue_len=64, batch_shift=1)
    want = oracle.build_graph_batched(x.cpu().numpy(), 32, prefix=2000, queue_len=64,
                                      batch_shift=1, nthreads=16)
    np.testing.assert_array_equal(got, want)


def test_batched_whole_prefix_is_song_build_graph():
    x = og._int_data(3000, 32, 11)
    np.testing.assert_array_equal(gbuild_batched(x, 16, prefix=3000), gbuild(x, 16))


@pytest.mark.parametrize("metric", ["ip", "cosine"])
def test_batched_float_metrics_search_well(metric):
    cfg = CONFIGS["glove200" if metric == "ip" else "nytimes256"]
    x, q = make_data(cfg, device="cuda", n=20_000, nq=200)
    s = song()
    adj = s.build_graph_batched(x, 32, metric, prefix=2000, queue_len=64)
    exact = s.build_graph(x, 32, metric)
    truth = oracle.bruteforce(x.cpu().numpy(), q.cpu().numpy(), 10,
                              metric=oracle.METRICS[metric])[0]
    rec = []
    for g in (adj, exact):
        idx = s.SongIndex(x, g, metric=metric)
        ids, _ = idx.search(q, params=s.Params(K=10, queue_len=256))
        rec.append(oracle.recall(ids.cpu().numpy(), truth))
        idx.close()
    assert rec[0] >= rec[1] - 0.05, rec


def test_batched_errors():
    s = song()
    x = torch.zeros((100, 8), device="cuda")
    for kw in (dict(prefix=0), dict(queue_len=4), dict(batch_shift=17)):
        with pytest.raises(s.SongError):
            s.build_graph_batched(x, 8, **kw)


def test_from_forward_bit_exact():
    """song_build_graph_from_forward (R15 steps 2-4 on given lists) against the
    oracle's, on the oracle's own exact forward lists and on lists with gaps."""
    x = og._int_data(2500, 24, 21)
    fi, fd = oracle.forward_lists(x, 16, nthreads=8)
    fi[::7, 5:] = -1  # shorter lists on some rows
    fd[::7, 5:] = np.inf
    want = oracle.build_graph_from_forward(x, fi, fd, nthreads=8)
    s = song()
    got = s.build_graph_from_forward(torch.as_tensor(x, device="cuda"),
                                     torch.as_tensor(fi, device="cuda"),
                                     torch.as_tensor(fd, device="cuda"))
    torch.cuda.synchronize()
    np.testing.assert_array_equal(got.cpu().numpy(), want)
    np.testing.assert_array_equal(oracle.build_graph_from_forward(x, *oracle.forward_lists(x, 16)),
                                  oracle.build_graph(x, 16))


def test_from_forward_knn_lists_bit_exact():
    """Unrestricted kNN lists (each row's D nearest of ALL rows, itself
    included at distance 0, mutual neighbours in both F and B): C(v) is taken
    as a set — no self loop, no repeated id — on the GPU as in the oracle."""
    x = og._int_data(1500, 16, 31)
    D = 12
    xn = x.astype(np.float64)
    d = ((xn[:, None, :] - xn[None, :, :]) ** 2).sum(-1)
    order = np.lexsort((np.broadcast_to(np.arange(len(x)), d.shape), d), axis=1)[:, :D]
    fi = order.astype(np.int32)
    fd = np.take_along_axis(d, order, 1).astype(np.float32)
    want = oracle.build_graph_from_forward(x, fi, fd, nthreads=8)
    s = song()
    got = s.build_graph_from_forward(torch.as_tensor(x, device="cuda"),
                                     torch.as_tensor(fi, device="cuda"),
                                     torch.as_tensor(fd, device="cuda")).cpu().numpy()
    np.testing.assert_array_equal(got, want)
    for v, row in enumerate(got):
        r = [int(j) for j in row if j >= 0]
        assert v not in r and len(set(r)) == len(r)


def test_builders_reject_bad_input():
    s = song()
    x = torch.randn(3000, 16, device="cuda")
    x[2999, 3] = float("nan")  # the last row: outside any exact prefix
    for build in (lambda: s.build_graph(x, 8),
                  lambda: s.build_graph_batched(x, 8, prefix=100, queue_len=32),
                  lambda: s.build_graph_batched(x, 8, prefix=5000, queue_len=32)):
        with pytest.raises(s.SongError) as e:
            build()
        assert e.value.code == -1
    x[2999, 3] = 0.0
    fi = torch.zeros((3000, 8), dtype=torch.int32, device="cuda")
    fd = torch.zeros((3000, 8), device="cuda")
    fi[5, 2] = 3000  # outside [-1, n)
    with pytest.raises(s.SongError) as e:
        s.build_graph_from_forward(x, fi, fd)
    assert e.value.code == -1


def test_tensor_core_path_only_when_exact(monkeypatch):
    """Non-integer data never takes the tensor-core Gram by default: the auto
    path gives the FFMA path's graph bit for bit."""
    rng = np.random.default_rng(9)
    x = (rng.integers(0, 200, (1500, 64)) / 8.0).astype(np.float32)  # tf32-representable, not integer
    auto = gbuild(x, 16)
    monkeypatch.setenv("SONG_GRAPH_PATH", "simt")
    np.testing.assert_array_equal(auto, gbuild(x, 16))


@pytest.mark.parametrize("take", [0, 1, 8, 31, 32])
def test_merge_graph_rows_bit_exact(take):
    """song_graph_merge_rows (reading R18) against the oracle's definition, on
    rows with padding, repeats inside a row and ids shared by both rows."""
    rng = np.random.default_rng(take)
    n, D = 3000, 32
    a = rng.integers(-1, 200, (n, D)).astype(np.int32)
    b = rng.integers(-1, 200, (n, D)).astype(np.int32)
    s = song()
    got = s.merge_graph_rows(torch.as_tensor(a, device="cuda"), torch.as_tensor(b, device="cuda"),
                             take).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.merge_graph_rows(a, b, take))
    for D2 in (7, 16):  # degrees below 32
        a2, b2 = a[:, :D2].copy(), b[:, :D2].copy()
        got = s.merge_graph_rows(torch.as_tensor(a2, device="cuda"),
                                 torch.as_tensor(b2, device="cuda"), min(take, D2)).cpu().numpy()
        np.testing.assert_array_equal(got, oracle.merge_graph_rows(a2, b2, min(take, D2)))
