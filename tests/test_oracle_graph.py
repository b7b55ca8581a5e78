"""Pins of the oracle's graph construction (reading R15; SONG loads NSW graphs,
P:477), CPU only: a hand-worked 6-point example, the forward lists
against a numpy brute force, the backward-list definition, structural
properties, and agreement with the independent torch tooling
(workloads/graph.py) on tie-free data."""
import numpy as np
import pytest

import oracle
from _golden import golden_path


def load_toy():
    coords, rows = {}, {}
    for line in open(golden_path("graph_toy.txt")):
        line = line.split("#", 1)[0].split()
        if not line:
            continue
        if line[0] == "coord":
            coords[int(line[1])] = float(line[2])
        elif line[0] == "row":
            rows[int(line[1])] = [int(x) for x in line[2:]]
    n = len(coords)
    x = np.array([[coords[i]] for i in range(n)], np.float32)
    adj = np.array([rows[i] for i in range(n)], np.int32)
    return x, adj


def test_hand_worked_example():
    x, want = load_toy()
    np.testing.assert_array_equal(oracle.build_graph(x, 2), want)


def _forward_bruteforce(x, D):
    n = len(x)
    d = ((x[:, None, :].astype(np.float64) - x[None, :, :]) ** 2).sum(-1).astype(np.float32)
    F = []
    for i in range(n):
        keys = sorted((d[i, j], j) for j in range(i))
        F.append(keys[:D])
    return d, F


@pytest.mark.parametrize("D", [2, 5, 8])
def test_rows_follow_the_definition(D):
    """Each row is a subset of F(v) u B(v), starts with the nearest candidate,
    has no repeats and is padded only when there are fewer than D candidates."""
    rng = np.random.default_rng(D)
    n = 300
    x = rng.integers(0, 50, (n, 3)).astype(np.float32)  # integer: exact, many ties
    adj = oracle.build_graph(x, D)
    d, F = _forward_bruteforce(x, D)
    B = [[] for _ in range(n)]
    for i in range(n):
        for dd, j in F[i]:
            B[j].append((dd, i))
    B = [sorted(b)[:D] for b in B]
    for v in range(n):
        C = sorted(F[v] + B[v])
        row = [int(u) for u in adj[v] if u >= 0]
        assert len(row) == len(set(row)) == min(D, len(C))
        assert set(row) <= {j for _, j in C}
        if C:
            assert row[0] == C[0][1]
        # a candidate left out while the row was still open was pruned: some
        # kept neighbour is at least as close to it as the base
        pos = {u: k for k, u in enumerate(row)}
        for t, (dc, c) in enumerate(C):
            if c not in pos and len(row) == D:
                kept_before = [u for u in row if (d[v, u], u) < (dc, c)]
                assert any(d[c, k] <= dc for k in kept_before) or len(kept_before) == D


def test_search_on_built_graph_full_queue_is_exact():
    rng = np.random.default_rng(11)
    x = rng.integers(0, 30, (400, 4)).astype(np.float32)
    adj = oracle.build_graph(x, 8)
    q = rng.integers(0, 30, (20, 4)).astype(np.float32)
    # entry 0 reaches everything: every i > 0 links back toward earlier ids or is linked
    ids, d, _, _ = oracle.search(x, adj, q, 5, 400)
    bi, bd = oracle.bruteforce(x, q, 5)
    np.testing.assert_array_equal(d, bd)


def test_agrees_with_the_torch_tooling():
    """workloads/graph.py implements the same construction with torch ops
    (GEMM distances, topk, argsort); on Gaussian data (no ties) the rows agree
    up to fp32-vs-fp64 near-ties."""
    import torch
    from workloads.graph import build_graph as tool_build
    rng = np.random.default_rng(5)
    x = rng.standard_normal((1500, 12)).astype(np.float32)
    a = oracle.build_graph(x, 16, nthreads=8)
    b = tool_build(torch.from_numpy(x), degree=16, row_block=512, col_block=4096).numpy()
    same_rows = (a == b).all(1).mean()
    same_sets = np.mean([set(r) == set(s) for r, s in zip(a, b)])
    assert same_sets >= 0.99 and same_rows >= 0.98


# ---------------------------------------------------------------- reading R16
def _int_data(n, dim, seed):
    rng = np.random.default_rng(seed)
    return rng.integers(0, 64, size=(n, dim)).astype(np.float32)


def test_forward_lists_match_bruteforce():
    x = _int_data(300, 8, 3)
    ids, dists = oracle.forward_lists(x, 6)
    for i, keys in enumerate(_forward_bruteforce(x, 6)[1]):
        assert [int(j) for j in ids[i] if j >= 0] == [j for _, j in keys]
        np.testing.assert_array_equal(dists[i, :len(keys)], [d for d, _ in keys])


def test_batched_with_whole_prefix_is_r15():
    """prefix >= n: no batches, R16 reduces to R15."""
    x = _int_data(400, 8, 4)
    np.testing.assert_array_equal(oracle.build_graph_batched(x, 8, prefix=400),
                                  oracle.build_graph(x, 8))


def test_batch_bounds():
    assert oracle.batch_bounds(10, 4, 1) == [(4, 6), (6, 9), (9, 10)]
    assert oracle.batch_bounds(10, 4, 0) == [(4, 8), (8, 10)]
    assert oracle.batch_bounds(3, 5, 1) == []


def test_batched_full_queue_equals_batch_restricted_definition():
    """With queue_len >= the searched prefix every search is exhaustive, so F(i)
    is the D nearest rows among those reachable from entry 0 in G_m (m = start
    of i's batch) — computed here by BFS + numpy brute force, independent of
    the oracle's search — and the graph is R15 steps 2-4 on those lists."""
    n, D, prefix, shift = 600, 6, 100, 1
    x = _int_data(n, 8, 5)
    d = ((x[:, None, :].astype(np.float64) - x[None, :, :]) ** 2).sum(-1).astype(np.float32)
    fi = np.full((n, D), -1, np.int32)
    fd = np.full((n, D), np.inf, np.float32)
    for i, keys in enumerate(_forward_bruteforce(x[:prefix], D)[1]):
        for t, (dd, j) in enumerate(keys):
            fi[i, t], fd[i, t] = j, dd
    for m, m1 in oracle.batch_bounds(n, prefix, shift):
        g = oracle.build_graph_from_forward(x[:m], fi[:m], fd[:m])
        seen, stack = {0}, [0]
        while stack:
            for u in g[stack.pop()]:
                if u >= 0 and int(u) not in seen:
                    seen.add(int(u))
                    stack.append(int(u))
        for i in range(m, m1):
            keys = sorted((d[i, j], j) for j in seen)[:D]
            for t, (dd, j) in enumerate(keys):
                fi[i, t], fd[i, t] = j, dd
    want = oracle.build_graph_from_forward(x, fi, fd)
    got = oracle.build_graph_batched(x, D, prefix=prefix, queue_len=n, batch_shift=shift)
    np.testing.assert_array_equal(got, want)


def test_batched_graph_is_valid_and_searchable():
    x = _int_data(2000, 16, 6)
    D = 8
    adj = oracle.build_graph_batched(x, D, prefix=200, queue_len=32, batch_shift=1)
    assert adj.shape == (2000, D)
    assert ((adj >= -1) & (adj < 2000)).all()
    for v, row in enumerate(adj):
        r = [int(j) for j in row if j >= 0]
        assert v not in r and len(set(r)) == len(r)
    q = _int_data(50, 16, 7)
    ids, _, _, _ = oracle.search(x, adj, q, 10, 64)
    truth, _ = oracle.bruteforce(x, q, 10)
    assert oracle.recall(ids, truth) > 0.9


def test_merge_graph_rows_definition():
    """Reading R18 on hand-worked rows: the first `take` of the IP row, then the
    angular row, then the rest of the IP row; ids once, -1 skipped, truncated."""
    first = np.array([[1, 2, 3, -1], [0, 2, 2, 5], [-1, -1, -1, -1]], np.int32)
    second = np.array([[3, 4, 5, 1], [5, 6, -1, 0], [7, -1, 8, 7]], np.int32)
    got = oracle.merge_graph_rows(first, second, 2)
    np.testing.assert_array_equal(got, [[1, 2, 3, 4], [0, 2, 5, 6], [7, 8, -1, -1]])
    # take 0 = the second graph first; take D = the first graph first
    np.testing.assert_array_equal(oracle.merge_graph_rows(first, second, 0)[0], [3, 4, 5, 1])
    np.testing.assert_array_equal(oracle.merge_graph_rows(first, second, 4)[1], [0, 2, 5, 6])
