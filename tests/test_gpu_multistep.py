"""GPU parity of multi-step probing (§V; reading R13): the kernel's
steps > 1 path against the oracle, bit-exact on integer-valued data (ids,
distances and counters), including candidate lists longer than one warp
(steps x degree up to 128, handled in groups of 32)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from workloads.graph import build_graph  # noqa: E402
from workloads.synth import CONFIGS, make_data  # noqa: E402

import test_oracle_pins as pins  # noqa: E402
from test_gpu_parity import song, gpu_search, assert_exact, small_random  # noqa: E402

FLAGS = {"hash": oracle.OPTIMIZED, "bloom": oracle.OPTIMIZED_BLOOM}


@pytest.mark.parametrize("visited", ["hash", "bloom"])
def test_toy_two_steps(visited):
    data, adj, _, _ = pins.load_toy()
    s = song()
    idx = s.SongIndex(data, adj)
    q = np.zeros((1, 1), np.float32)
    g = gpu_search(idx, q, 3, 3, visited, steps=2)
    o = oracle.search(data, adj, q, 3, 3, flags=FLAGS[visited], steps=2)
    assert_exact(g, o)
    assert [int(x) + 1 for x in g[0][0]] == [8, 2, 7]
    idx.close()


@pytest.fixture(scope="module")
def sift50k():
    cfg = CONFIGS["sift1m"]
    x, q = make_data(cfg, device="cuda", n=50_000, nq=300)
    adj = build_graph(x, degree=32)
    return cfg, x.cpu().numpy(), q.cpu().numpy(), adj.cpu().numpy()


@pytest.mark.parametrize("steps", [2, 3, 4])
@pytest.mark.parametrize("L", [10, 32, 64, 128, 200, 512])
@pytest.mark.parametrize("visited", ["hash", "bloom"])
def test_sift_multistep_bit_exact(sift50k, steps, L, visited):
    cfg, x, q, adj = sift50k
    s = song()
    idx = s.SongIndex(x, adj)
    g = gpu_search(idx, q, cfg.K, L, visited, steps=steps)
    o = oracle.search(x, adj, q, cfg.K, L, flags=FLAGS[visited], steps=steps, nthreads=8)
    assert_exact(g, o)
    idx.close()


@pytest.mark.parametrize("dim", [3, 130])
@pytest.mark.parametrize("L,K", [(1, 1), (33, 10), (150, 20)])
def test_multistep_edges(dim, L, K):
    """padding, repeated ids in a row (dedup within and across popped rows)."""
    x, adj, q = small_random(dim=dim)
    s = song()
    idx = s.SongIndex(x, adj)
    for steps in (2, 4):
        g = gpu_search(idx, q, K, L, "hash", steps=steps)
        o = oracle.search(x, adj, q, K, L, flags=oracle.OPTIMIZED, steps=steps)
        assert_exact(g, o)
    idx.close()


def test_multistep_errors(sift50k):
    cfg, x, q, adj = sift50k
    s = song()
    idx = s.SongIndex(x[:1000], np.clip(adj[:1000], -1, 999))
    qt = torch.as_tensor(q[:4], device="cuda")
    for kw, code in ((dict(steps=5), -4), (dict(steps=-1), -1),
                     (dict(steps=2, visited="cuckoo"), -4),
                     (dict(steps=2, visited="hashtable"), -4)):
        with pytest.raises(s.SongError) as e:
            idx.search(qt, params=s.Params(K=1, queue_len=8, **kw))
        assert e.value.code == code
    idx.close()
