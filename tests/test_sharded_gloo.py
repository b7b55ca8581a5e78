"""Multi-process (world size 2, gloo, CPU) tests of the sharding host logic.

The per-shard searcher is the oracle and the merger is the oracle's plain merge
definition, so these tests cover the orchestration (broadcast, id offsets,
all-gather, merge) without a GPU; the CUDA searcher/merger are exercised by
tests/test_gpu_parity.py::test_dataset_sharding_emulated_on_one_gpu.
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _problem():
    rng = np.random.default_rng(42)
    n, dim, nq, K, L = 1200, 6, 40, 10, 32
    x = rng.integers(0, 30, (n, dim)).astype(np.float32)
    q = rng.integers(0, 30, (nq, dim)).astype(np.float32)
    return x, q, K, L


def _shard_graph(xs):
    sys.path.insert(0, ROOT)
    from workloads.graph import build_graph
    return build_graph(torch.from_numpy(xs), degree=8, row_block=512, col_block=4096).numpy()


def _oracle_searcher(xs, adj, K, L):
    import oracle

    def run(q, id_offset):
        ids, d, _, _ = oracle.search(xs, adj, q.numpy(), K, L)
        ids = np.where(ids >= 0, ids + id_offset, -1)
        return torch.from_numpy(ids.astype(np.int32)), torch.from_numpy(d)
    return run


def _oracle_merger(K):
    import oracle

    def run(gi, gd):
        i, d = oracle.merge_shards(list(gi.numpy()), list(gd.numpy()), K)
        return torch.from_numpy(i), torch.from_numpy(d)
    return run


def _worker(rank, world, port, out_dir):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icde_zhaotl20_b200 import sharded
    x, q, K, L = _problem()
    lo, hi = sharded.shard_ranges(len(x), world)[rank]
    xs = x[lo:hi]
    adj = _shard_graph(xs)
    ids, dists = sharded.dataset_sharded_search(
        _oracle_searcher(xs, adj, K, L), _oracle_merger(K),
        torch.from_numpy(q) if rank == 0 else None, len(q), q.shape[1], K, lo,
        torch.device("cpu"))
    np.save(os.path.join(out_dir, f"ds_{rank}.npy"), np.stack([ids.numpy().astype(np.float64),
                                                              dists.numpy().astype(np.float64)]))
    # query sharding: replicated index (full graph), each rank its slice
    full_adj = np.load(os.path.join(out_dir, "full_adj.npy"))
    a, b = sharded.query_slice(len(q), rank, world)
    ids_q, d_q = sharded.query_sharded_search(_oracle_searcher(x, full_adj, K, L),
                                              torch.from_numpy(q[a:b]), gather=True)
    np.save(os.path.join(out_dir, f"qs_{rank}.npy"), np.stack([ids_q.numpy().astype(np.float64),
                                                              d_q.numpy().astype(np.float64)]))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_sharding_world2_gloo(tmp_path, world):
    import oracle
    from paper_conf_icde_zhaotl20_b200 import sharded
    x, q, K, L = _problem()
    full_adj = _shard_graph(x)
    np.save(tmp_path / "full_adj.npy", full_adj)
    mp.start_processes(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world,
                       join=True, start_method="spawn")
    # expected: per-shard oracle search in one process, merged by the definition
    per_i, per_d = [], []
    for lo, hi in sharded.shard_ranges(len(x), world):
        xs = x[lo:hi]
        i, d, _, _ = oracle.search(xs, _shard_graph(xs), q, K, L)
        per_i.append(np.where(i >= 0, i + lo, -1))
        per_d.append(d)
    ei, ed = oracle.merge_shards(per_i, per_d, K)
    for r in range(world):
        got = np.load(tmp_path / f"ds_{r}.npy")
        np.testing.assert_array_equal(got[0].astype(np.int32), ei)
        np.testing.assert_array_equal(got[1].astype(np.float32), ed)
    # merged shards still find true neighbours
    bi, _ = oracle.bruteforce(x, q, K)
    assert oracle.recall(ei, bi) > 0.9
    # query sharding == one process over the whole batch
    oi, od, _, _ = oracle.search(x, full_adj, q, K, L)
    for r in range(world):
        got = np.load(tmp_path / f"qs_{r}.npy")
        np.testing.assert_array_equal(got[0].astype(np.int32), oi)
        np.testing.assert_array_equal(got[1].astype(np.float32), od)


def test_shard_ranges_cover_exactly():
    from paper_conf_icde_zhaotl20_b200 import sharded
    for n in (1, 7, 100, 1001):
        for w in (1, 2, 3, 8):
            r = sharded.shard_ranges(n, w)
            assert r[0][0] == 0 and r[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(r, r[1:]))
            assert max(h - l for l, h in r) - min(h - l for l, h in r) <= 1
