"""SONG oracle — TEST INFRASTRUCTURE ONLY.

A plain CPU implementation of the search SONG accelerates (Algorithm 1 of
PAPER.md, with the §IV optimizations as switches), written from the
paper.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_icde_zhaotl20_b200`` never imports it and shares
no code with it (the C++ source is ``oracle/song_oracle.cpp``; the readings
R1-R16 it follows are listed in its header and in DESIGN.md §3).

This module only marshals numpy arrays into ``liboracle.so`` (built by
:func:`build`) and adds the two plain definitions the paper states in prose:
recall and the merge of per-shard results, plus the batch
loop of reading R16 (:func:`build_graph_batched`), which composes the C++
forward lists, graph steps and search in the order the reading states.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Callable, Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "song_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

L2, IP, COSINE, HAMMING = 0, 1, 2, 3
METRICS = {"l2": L2, "ip": IP, "cosine": COSINE, "hamming": HAMMING}

# Mode flags (must match song_oracle.cpp's enum Flags).
PLAIN = 0
BOUNDED_Q = 1
SEL = 2
DEL = 4
BLOOM = 8
CUCKOO = 16
LAZY = 32   # with DEL: deletions deferred until visited reaches lazy_cap (reading R14)
OPTIMIZED = BOUNDED_Q | SEL | DEL          # "hashtable-sel-del" (Fig. 7)
OPTIMIZED_BLOOM = BOUNDED_Q | SEL | BLOOM  # "bloomfilter" (Fig. 7)
OPTIMIZED_CUCKOO = BOUNDED_Q | SEL | DEL | CUCKOO  # "cuckoofilter" (Fig. 7)
HASHTABLE = BOUNDED_Q                      # "hashtable" (Fig. 7): no sel, no del
HASHTABLE_SEL = BOUNDED_Q | SEL            # "hashtable-sel" (Fig. 7)
OPTIMIZED_LAZY = OPTIMIZED | LAZY          # hash-sel-del with lazy deletion (R14)
UNION = 64  # q and topk as one bounded list of the L best discovered keys (reading R17)
OPTIMIZED_UNION = OPTIMIZED | UNION
OPTIMIZED_UNION_LAZY = OPTIMIZED_LAZY | UNION

_TRACE_FN = ctypes.CFUNCTYPE(
    None, ctypes.c_void_p, ctypes.c_int64,
    ctypes.POINTER(ctypes.c_int32), ctypes.c_int64,
    ctypes.POINTER(ctypes.c_int32), ctypes.c_int64,
    ctypes.POINTER(ctypes.c_int32), ctypes.c_int64)

_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (plain -O2, no vectorisation tricks)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-o", _LIB, _SRC]
        subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        lib.oracle_search.restype = ctypes.c_int64
        lib.oracle_search.argtypes = [
            P, ctypes.c_int64, ctypes.c_int32, P, ctypes.c_int32, ctypes.c_int32,
            P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
            ctypes.c_int64, ctypes.c_int32, ctypes.c_int64, P, P, P,
            ctypes.c_int32, _TRACE_FN, P]
        lib.oracle_search_steps.restype = ctypes.c_int64
        lib.oracle_search_steps.argtypes = [
            P, ctypes.c_int64, ctypes.c_int32, P, ctypes.c_int32, ctypes.c_int32,
            P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
            ctypes.c_int64, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_int64,
            P, P, P, ctypes.c_int32, _TRACE_FN, P]
        lib.oracle_distance.restype = ctypes.c_float
        lib.oracle_distance.argtypes = [P, P, ctypes.c_int32, ctypes.c_int32]
        lib.oracle_bruteforce.restype = None
        lib.oracle_bruteforce.argtypes = [P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                          P, ctypes.c_int64, ctypes.c_int32, P, P, ctypes.c_int32]
        lib.oracle_cuckoo_probe.restype = ctypes.c_int64
        lib.oracle_cuckoo_probe.argtypes = [ctypes.c_int64, P, ctypes.c_int64, P,
                                            ctypes.c_int64, P]
        lib.oracle_rp_encode.restype = None
        lib.oracle_rp_encode.argtypes = [P, ctypes.c_int64, ctypes.c_int32, P, ctypes.c_int32, P,
                                         ctypes.c_int32]
        lib.oracle_forward_lists.restype = None
        lib.oracle_forward_lists.argtypes = [P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                             ctypes.c_int32, P, P, ctypes.c_int32]
        lib.oracle_build_graph_from_forward.restype = None
        lib.oracle_build_graph_from_forward.argtypes = [P, ctypes.c_int64, ctypes.c_int32,
                                                        ctypes.c_int32, ctypes.c_int32, P, P, P,
                                                        ctypes.c_int32]
        lib.oracle_build_graph.restype = None
        lib.oracle_build_graph.argtypes = [P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                           ctypes.c_int32, P, ctypes.c_int32]
        lib.oracle_bloom_probe.restype = None
        lib.oracle_bloom_probe.argtypes = [ctypes.c_int64, P, ctypes.c_int64, P,
                                           ctypes.c_int64, P]
        _lib = lib
    return _lib


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def default_cuckoo_buckets(L: int) -> int:
    """DESIGN.md reading R10: 4-slot buckets, >= 4x the live bound 2L + 32."""
    slots = 1 << int(np.ceil(np.log2(4 * (2 * L + 32))))
    return slots // 4


def cuckoo_probe(buckets: int, ops, probes):
    """Apply ops (id >= 0 insert, -(id+1) erase) then probe membership."""
    lib = _load()
    o = np.ascontiguousarray(ops, np.int64)
    pr = _i32(probes)
    out = np.empty(pr.shape[0], np.uint8)
    drops = lib.oracle_cuckoo_probe(int(buckets), _ptr(o), o.shape[0], _ptr(pr), pr.shape[0],
                                    _ptr(out))
    return out.astype(bool), int(drops)


def default_bloom_bits(L: int) -> int:
    """DESIGN.md reading A11: m = 2^ceil(log2(10 * 8L)) bits."""
    need = 10 * 8 * L
    return 1 << int(np.ceil(np.log2(need)))


def search(data, adj, queries, K: int, L: int, metric: int = L2, flags: int = OPTIMIZED,
           bloom_bits: Optional[int] = None, entry: int = 0, max_iters: int = 1 << 40,
           nthreads: int = 1, trace: Optional[Callable] = None, steps: int = 1,
           lazy_cap: int = 0):
    """Run the oracle.  Returns (ids [nq,K] int32, dists [nq,K] f32,
    counters [nq,2] int64 = (n_dist, n_exp), n_capped).  ``bloom_bits`` is the
    Bloom filter's bit count, or the Cuckoo filter's bucket count; ``steps`` is
    the multi-step probing width (pops per iteration, reading R13); ``lazy_cap``
    the visited capacity of the LAZY flag (reading R14)."""
    lib = _load()
    data = _f32(data)
    adj = _i32(adj)
    queries = _f32(queries)
    if queries.ndim == 1:
        queries = queries[None, :]
    n, dim = data.shape
    degree = adj.shape[1]
    nq = queries.shape[0]
    assert adj.shape[0] == n and queries.shape[1] == dim
    assert 1 <= K <= L
    ids = np.empty((nq, K), np.int32)
    dists = np.empty((nq, K), np.float32)
    counters = np.empty((nq, 2), np.int64)
    if bloom_bits is None:
        bloom_bits = default_cuckoo_buckets(L) if flags & CUCKOO else default_bloom_bits(L)
    cb = _TRACE_FN()
    if trace is not None:
        def _cb(ctx, it, qp, nqq, tp, nt, vp, nv):
            q_ids = [qp[i] for i in range(nqq)]
            t_ids = [tp[i] for i in range(nt)]
            v_ids = None if nv < 0 else [vp[i] for i in range(nv)]
            trace(int(it), q_ids, t_ids, v_ids)
        cb = _TRACE_FN(_cb)
    capped = lib.oracle_search_steps(_ptr(data), n, dim, _ptr(adj), degree, metric,
                                     _ptr(queries), nq, K, L, flags, int(bloom_bits), entry,
                                     int(max_iters), int(steps), int(lazy_cap), _ptr(ids),
                                     _ptr(dists),
                                     _ptr(counters), int(nthreads), cb, None)
    return ids, dists, counters, int(capped)


def distance(p, x, metric: int = L2) -> float:
    lib = _load()
    p = _f32(p)
    x = _f32(x)
    return float(lib.oracle_distance(_ptr(p), _ptr(x), p.shape[0], metric))


def bruteforce(data, queries, K: int, metric: int = L2, nthreads: int = 1):
    """Exact top-K under the (dist, id) order — recall ground truth B."""
    lib = _load()
    data = _f32(data)
    queries = _f32(queries)
    if queries.ndim == 1:
        queries = queries[None, :]
    n, dim = data.shape
    nq = queries.shape[0]
    ids = np.empty((nq, K), np.int32)
    dists = np.empty((nq, K), np.float32)
    lib.oracle_bruteforce(_ptr(data), n, dim, metric, _ptr(queries), nq, K, _ptr(ids),
                          _ptr(dists), int(nthreads))
    return ids, dists


def bloom_probe(bits: int, inserted, probes):
    lib = _load()
    ins = _i32(inserted)
    pr = _i32(probes)
    out = np.empty(pr.shape[0], np.uint8)
    lib.oracle_bloom_probe(int(bits), _ptr(ins), ins.shape[0], _ptr(pr), pr.shape[0], _ptr(out))
    return out.astype(bool)


def rp_encode(data, R, nthreads: int = 1):
    """1-bit random projection (§VII; reading R11): codes [n, h/32]
    uint32, bit j = [<x, r_j> > 0] accumulated in fp64, LSB-first packing.
    ``R`` is [h, dim] (row j = r_j); h % 32 == 0."""
    lib = _load()
    data = _f32(data)
    R = _f32(R)
    n, dim = data.shape
    h = R.shape[0]
    assert R.shape[1] == dim and h % 32 == 0 and h > 0
    codes = np.empty((n, h // 32), np.uint32)
    lib.oracle_rp_encode(_ptr(data), n, dim, _ptr(R), h, _ptr(codes), int(nthreads))
    return codes


def _codes_as_f32(codes):
    c = np.ascontiguousarray(codes, dtype=np.uint32)
    if c.ndim == 1:
        c = c[None, :]
    return c.view(np.float32)


def search_codes(codes, adj, qcodes, K: int, L: int, flags: int = OPTIMIZED, **kw):
    """Algorithm 1 over h-bit codes with the Hamming distance (reading R12).
    codes [n, h/32] / qcodes [nq, h/32] uint32; returns as :func:`search`."""
    return search(_codes_as_f32(codes), adj, _codes_as_f32(qcodes), K, L, metric=HAMMING,
                  flags=flags, **kw)


def bruteforce_codes(codes, qcodes, K: int, nthreads: int = 1):
    """Exact top-K under (Hamming distance, id)."""
    return bruteforce(_codes_as_f32(codes), _codes_as_f32(qcodes), K, metric=HAMMING,
                      nthreads=nthreads)


def hamming(a, b) -> int:
    """Hamming distance of two codes through the oracle's R12 routine."""
    return int(distance(_codes_as_f32(a)[0], _codes_as_f32(b)[0], HAMMING))


def code_bytes(n: int, h: int) -> int:
    """Table IV: an h-bit code takes h/32 words = h/8 bytes per point."""
    return n * h // 8


def build_graph(data, degree: int, metric: int = L2, nthreads: int = 1):
    """Graph construction of reading R15 (exact-insertion NSW forward lists,
    capped backward lists, HNSW heuristic with refill): adjacency [n, degree]
    int32, -1 padded."""
    lib = _load()
    data = _f32(data)
    n, dim = data.shape
    adj = np.empty((n, degree), np.int32)
    lib.oracle_build_graph(_ptr(data), n, dim, metric, degree, _ptr(adj), int(nthreads))
    return adj


def forward_lists(data, degree: int, metric: int = L2, nthreads: int = 1):
    """R15 step 1 alone: the exact-insertion forward lists F(i) = the `degree`
    smallest (d(i, j), j), j < i, as (ids, dists) [n, degree] (-1 / +inf pad)."""
    lib = _load()
    data = _f32(data)
    n, dim = data.shape
    ids = np.empty((n, degree), np.int32)
    dists = np.empty((n, degree), np.float32)
    lib.oracle_forward_lists(_ptr(data), n, dim, metric, degree, _ptr(ids), _ptr(dists),
                             int(nthreads))
    return ids, dists


def build_graph_from_forward(data, fwd_ids, fwd_dists, metric: int = L2, nthreads: int = 1):
    """R15 steps 2-4 (backward lists, candidates, heuristic with refill) on the
    given forward lists (ids / dists [n, degree], -1 padded, ascending keys)."""
    lib = _load()
    data = _f32(data)
    fwd_ids = _i32(fwd_ids)
    fwd_dists = _f32(fwd_dists)
    n, dim = data.shape
    degree = fwd_ids.shape[1]
    adj = np.empty((n, degree), np.int32)
    lib.oracle_build_graph_from_forward(_ptr(data), n, dim, metric, degree, _ptr(fwd_ids),
                                        _ptr(fwd_dists), _ptr(adj), int(nthreads))
    return adj


def batch_bounds(n: int, prefix: int, batch_shift: int):
    """Reading R16's insertion batches: [m, m + max(1, m >> batch_shift)) from
    m = min(n, prefix) until n."""
    m = min(n, max(1, prefix))
    out = []
    while m < n:
        b = min(n - m, max(1, m >> batch_shift))
        out.append((m, m + b))
        m += b
    return out


def build_graph_batched(data, degree: int, metric: int = L2, prefix: int = 65536,
                        queue_len: int = 64, batch_shift: int = 1, nthreads: int = 1):
    """Reading R16, batched-insertion NSW (the scale-out builder), step by step:
    1. F(i) for i < prefix: R15's exact forward lists;
    2. for each batch [m, m'): G_m = R15 steps 2-4 on F of rows [0, m); every
       i in the batch searches G_m (Algorithm 1 from entry 0, K = degree,
       L = queue_len) and F(i) = the search's top `degree` (ids < m);
    3. the graph = R15 steps 2-4 on all of F."""
    data = _f32(data)
    n = data.shape[0]
    D = degree
    m0 = min(n, max(1, prefix))
    fi = np.full((n, D), -1, np.int32)
    fd = np.full((n, D), np.inf, np.float32)
    fi[:m0], fd[:m0] = forward_lists(data[:m0], D, metric, nthreads)
    for m, m1 in batch_bounds(n, prefix, batch_shift):
        g = build_graph_from_forward(data[:m], fi[:m], fd[:m], metric, nthreads)
        ids, dists, _, _ = search(data[:m], g, data[m:m1], D, max(queue_len, D), metric=metric,
                                  flags=OPTIMIZED, nthreads=nthreads)
        fi[m:m1], fd[m:m1] = ids, dists
    return build_graph_from_forward(data, fi, fd, metric, nthreads)


def recall(found_ids, truth_ids) -> float:
    """Mean over queries of |A ∩ B| / |B|; B = truth_ids rows."""
    found_ids = np.asarray(found_ids)
    truth_ids = np.asarray(truth_ids)
    tot = 0.0
    for a, b in zip(found_ids, truth_ids):
        bs = set(int(x) for x in b if x >= 0)
        if not bs:
            continue
        tot += len(bs & set(int(x) for x in a if x >= 0)) / len(bs)
    return tot / max(1, len(truth_ids))


def merge_shards(ids_per_shard, dists_per_shard, K: int):
    """P:471 "perform graph search on each GPU and merge the results": the
    plain definition — concatenate every shard's (dist, global id) list and keep
    the K smallest under the (dist, id) order (R2)."""
    ids = np.concatenate([np.asarray(x) for x in ids_per_shard], axis=1)
    dists = np.concatenate([np.asarray(x) for x in dists_per_shard], axis=1)
    nq = ids.shape[0]
    out_i = np.full((nq, K), -1, np.int32)
    out_d = np.full((nq, K), np.inf, np.float32)
    for r in range(nq):
        pairs = sorted((float(d), int(i)) for d, i in zip(dists[r], ids[r]) if i >= 0)
        for j, (d, i) in enumerate(pairs[:K]):
            out_i[r, j] = i
            out_d[r, j] = d
    return out_i, out_d


def merge_graph_rows(first, second, take_first: int):
    """Reading R18, written out: row v = first[v][:take], then second[v], then
    first[v][take:], each id once (first occurrence), -1 skipped, truncated to
    the degree, -1 padded."""
    first = np.asarray(first)
    second = np.asarray(second)
    n, D = first.shape
    out = np.full((n, D), -1, np.int32)
    for v in range(n):
        seq = list(first[v][:take_first]) + list(second[v]) + list(first[v][take_first:])
        kept = []
        for i in seq:
            if i >= 0 and i not in kept:
                kept.append(int(i))
        kept = kept[:D]
        out[v, :len(kept)] = kept
    return out
