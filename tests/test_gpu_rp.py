"""GPU parity of §VII: the 1-bit random-projection encoder and the
Hamming-distance search, through the C ABI, against the oracle.

Bars: codes bit-exact on the workload's certified-exact recipe (integer
pixels, 1/64-step R: tests/test_oracle_rp.py::test_rp_recipe_is_exact_in_fp32);
on generic float data a differing bit must sit on a projection within fp32
rounding of 0.  Search over codes: ids, Hamming distances and counters
bit-exact (integer arithmetic end to end).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from workloads.graph import build_graph  # noqa: E402
from workloads.synth import MnistLike, rp_matrix  # noqa: E402


def song():
    from paper_conf_icde_zhaotl20_b200 import song as s
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return s


def as_u32(t):
    return t.cpu().numpy().view(np.uint32)


@pytest.fixture(scope="module")
def mnist():
    gen = MnistLike(784, 600)
    x = gen.sample(6000, 600)
    q = gen.sample(300, 601)
    adj = build_graph(x.cuda(), degree=32).cpu().numpy()
    return x.numpy(), q.numpy(), adj


@pytest.mark.parametrize("bits", [32, 64, 96, 128, 256, 512, 1024])
def test_encoder_bit_exact_on_certified_recipe(mnist, bits):
    x, _, _ = mnist
    R = rp_matrix(bits, 784, 603 + bits).numpy()
    g = song().rp_encode(torch.as_tensor(x[:1333], device="cuda"), torch.as_tensor(R))
    torch.cuda.synchronize()
    np.testing.assert_array_equal(as_u32(g), oracle.rp_encode(x[:1333], R, nthreads=8))


@pytest.mark.parametrize("n,dim", [(1, 1), (129, 3), (300, 17), (257, 200), (1000, 960)])
def test_encoder_generic_float_data(n, dim):
    """Gaussian data and R: bits may differ only where |<x, r>| is within fp32
    accumulation error of 0 (the sign is decided in fp32 on the GPU, fp64 in
    the oracle)."""
    rng = np.random.default_rng(n * 7 + dim)
    x = rng.standard_normal((n, dim)).astype(np.float32)
    R = rng.standard_normal((128, dim)).astype(np.float32)
    g = as_u32(song().rp_encode(torch.as_tensor(x, device="cuda"), torch.as_tensor(R)))
    torch.cuda.synchronize()
    o = oracle.rp_encode(x, R)
    diff = np.unpackbits((g ^ o).view(np.uint8), bitorder="little").reshape(n, 128).astype(bool)
    proj = x.astype(np.float64) @ R.astype(np.float64).T
    bound = 4 * dim * np.finfo(np.float32).eps * (np.abs(x).astype(np.float64) @ np.abs(R).T)
    assert np.all(np.abs(proj[diff]) <= bound[diff])
    assert diff.mean() < 1e-3


@pytest.mark.parametrize("bits", [32, 128, 512])
@pytest.mark.parametrize("L", [1, 10, 32, 64, 100, 128, 256])
@pytest.mark.parametrize("visited", ["hash", "bloom"])
def test_hamming_search_bit_exact(mnist, bits, L, visited):
    x, q, adj = mnist
    R = rp_matrix(bits, 784, 603).numpy()
    codes = oracle.rp_encode(x, R, nthreads=8)
    qc = oracle.rp_encode(q, R, nthreads=8)
    s = song()
    idx = s.SongIndex.from_codes(codes, bits, adj)
    K = min(L, 10)
    ids, d, c = idx.search_codes(torch.as_tensor(qc.view(np.int32), device="cuda"),
                                 s.Params(K=K, queue_len=L, visited=visited), counters=True)
    torch.cuda.synchronize()
    idx.last_status()
    from test_gpu_parity import oracle_kw
    oi, od, oc, _ = oracle.search_codes(codes, adj, qc, K, L, nthreads=8, **oracle_kw(visited, L, idx=idx))
    np.testing.assert_array_equal(ids.cpu().numpy(), oi)
    np.testing.assert_array_equal(d.cpu().numpy(), od)
    np.testing.assert_array_equal(c.cpu().numpy().astype(np.int64), oc)
    idx.close()


@pytest.mark.parametrize("chunk_rows", ["0", "1000"])
def test_rp_index_end_to_end(mnist, monkeypatch, chunk_rows):
    """song_index_create_rp streams host vectors through the encoder in chunks
    (P:465); song_search_ex / song_search encode float queries with the same R.
    Equal to oracle.rp_encode + oracle.search_codes bit for bit."""
    if chunk_rows != "0":
        monkeypatch.setenv("SONG_RP_CHUNK_ROWS", chunk_rows)
    x, q, adj = mnist
    bits = 128
    R = rp_matrix(bits, 784, 603).numpy()
    s = song()
    idx = s.SongIndex.from_rp(x, R, adj)
    info = idx.info()
    assert (info.code_bits, info.dim, info.dim_padded, info.metric) == (128, 784, 4, 3)
    assert info.vector_bytes == x.shape[0] * bits // 8  # Table IV layout
    ids, d, c = idx.search(torch.as_tensor(q, device="cuda"),
                           params=s.Params(K=1, queue_len=64), counters=True)
    torch.cuda.synchronize()
    idx.last_status()
    codes = oracle.rp_encode(x, R, nthreads=8)
    qc = oracle.rp_encode(q, R, nthreads=8)
    from test_gpu_parity import oracle_kw
    oi, od, oc, _ = oracle.search_codes(codes, adj, qc, 1, 64, nthreads=8, **oracle_kw("hash", 64, idx=idx))
    np.testing.assert_array_equal(ids.cpu().numpy(), oi)
    np.testing.assert_array_equal(d.cpu().numpy(), od)
    np.testing.assert_array_equal(c.cpu().numpy().astype(np.int64), oc)
    hi, hd = idx.search_host(q[:77], 1, 64)  # song_search: host buffers
    np.testing.assert_array_equal(hi, oi[:77])
    np.testing.assert_array_equal(hd, od[:77])
    idx.close()


def test_hamming_errors(mnist):
    x, q, adj = mnist
    s = song()
    codes = np.zeros((x.shape[0], 4), np.uint32)
    idx = s.SongIndex.from_codes(codes, 128, adj)
    with pytest.raises(s.SongError) as e:  # a codes-only index takes codes
        idx.search(torch.zeros((2, 784), device="cuda"), params=s.Params(K=1, queue_len=8))
    assert e.value.code == -1
    with pytest.raises(s.SongError) as e:
        idx.search_codes(torch.zeros((2, 4), dtype=torch.int32, device="cuda"),
                         s.Params(K=1, queue_len=8, visited="cuckoo"))
    assert e.value.code == -4
    # all-equal codes: every distance 0, ties broken by id (reading A3)
    ids, d = idx.search_codes(torch.zeros((2, 4), dtype=torch.int32, device="cuda"),
                              s.Params(K=5, queue_len=16))
    torch.cuda.synchronize()
    assert (d.cpu().numpy() == 0).all()
    oi, od, _, _ = oracle.search_codes(codes, adj, np.zeros((2, 4), np.uint32), 5, 16)  # ids only
    np.testing.assert_array_equal(ids.cpu().numpy(), oi)
    idx.close()


@pytest.mark.parametrize("bits", [32, 64, 96, 128, 160, 256])
def test_code_footprint_is_table4s(mnist, bits):
    """Table IV: h/8 bytes per point (h = 96 / 160 round up to 16 B)."""
    x, q, adj = mnist
    R = rp_matrix(bits, 784, 603).numpy()
    codes = oracle.rp_encode(x, R, nthreads=8)
    qc = oracle.rp_encode(q[:50], R)
    s = song()
    idx = s.SongIndex.from_codes(codes, bits, adj)
    info = idx.info()
    words = bits // 32
    padded = words if words <= 2 else (words + 3) // 4 * 4
    assert info.vector_bytes == x.shape[0] * padded * 4
    if bits in (32, 64, 128, 256):
        assert info.vector_bytes == x.shape[0] * bits // 8
    ids, d, c = idx.search_codes(torch.as_tensor(qc.view(np.int32), device="cuda"),
                                 s.Params(K=5, queue_len=40), counters=True)
    torch.cuda.synchronize()
    from test_gpu_parity import oracle_kw
    oi, od, oc, _ = oracle.search_codes(codes, adj, qc, 5, 40, **oracle_kw("hash", 40, idx=idx))
    np.testing.assert_array_equal(ids.cpu().numpy(), oi)
    np.testing.assert_array_equal(d.cpu().numpy(), od)
    np.testing.assert_array_equal(c.cpu().numpy().astype(np.int64), oc)
    idx.close()
