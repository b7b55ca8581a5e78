"""Thin Python binding of libsong.so (include/song.h): argument marshalling only.

Every step of the search runs in the sm_100a kernels behind the C ABI; this
module never computes a distance, a queue or a visited set, and there is no
CPU fallback: if libsong.so or a CUDA device is missing, calls raise.

torch is used only for device memory and streams: CUDA tensors are passed to
``song_search_ex`` as raw device pointers on torch's current stream.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional, Tuple

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SONG_LIB", os.path.join(_PKG, "libsong.so"))

L2, IP, COSINE, HAMMING = 0, 1, 2, 3
METRICS = {"l2": L2, "ip": IP, "cosine": COSINE, "hamming": HAMMING}
VISITED_HASH, VISITED_BLOOM, VISITED_HASH_GLOBAL, VISITED_HASH_GLOBAL_SEL, VISITED_CUCKOO = range(5)
# names follow the paper's Fig. 7 legend
VISITED = {"hash": VISITED_HASH, "bloom": VISITED_BLOOM, "hashtable": VISITED_HASH_GLOBAL,
           "hashtable-sel": VISITED_HASH_GLOBAL_SEL, "cuckoo": VISITED_CUCKOO}

STATUS = {0: "SONG_OK", -1: "SONG_EINVAL", -2: "SONG_ENOMEM", -3: "SONG_ECUDA",
          -4: "SONG_EUNSUPPORTED", -5: "SONG_EITERCAP"}

EXPORTED = ["song_default_params", "song_index_create", "song_index_create_device",
            "song_index_destroy", "song_index_get_info", "song_search", "song_search_ex", "song_search_pipelined",
            "song_index_last_status", "song_merge_topk", "song_last_error", "song_version",
            "song_rp_encode", "song_index_create_codes", "song_index_create_rp",
            "song_search_codes_ex", "song_build_graph", "song_build_graph_batched", "song_build_graph_from_forward",
            "song_search_plan_get", "song_stage_cycles", "song_merge_topk_peers",
            "song_graph_merge_rows"]


class SongError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


SCHEDULES = {"auto": 0, "batch": 1, "outlier_first": 2}  # song.h SONG_SCHEDULE_*
QUEUE_KINDS = {"auto": 0, "separate": 1, "union": 2}     # song.h SONG_QUEUE_*


class SearchParams(ctypes.Structure):
    _fields_ = [("K", ctypes.c_int32), ("queue_len", ctypes.c_int32),
                ("visited", ctypes.c_int32), ("bloom_log2_bits", ctypes.c_int32),
                ("entry", ctypes.c_int32), ("max_iters", ctypes.c_int32),
                ("warps_per_block", ctypes.c_int32), ("blocks_per_sm", ctypes.c_int32),
                ("id_offset", ctypes.c_int32), ("table_log2", ctypes.c_int32),
                ("steps", ctypes.c_int32), ("visited_cap", ctypes.c_int32),
                ("schedule", ctypes.c_int32), ("queue_kind", ctypes.c_int32),
                ("queries_per_warp", ctypes.c_int32)]


class IndexInfo(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("dim", ctypes.c_int32), ("dim_padded", ctypes.c_int32),
                ("degree", ctypes.c_int32), ("metric", ctypes.c_int32),
                ("vector_bytes", ctypes.c_int64), ("graph_bytes", ctypes.c_int64),
                ("device", ctypes.c_int32), ("num_sms", ctypes.c_int32),
                ("code_bits", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class SearchPlan(ctypes.Structure):
    _fields_ = [("visited_log2", ctypes.c_int32), ("visited_cap", ctypes.c_int32),
                ("queue_regs", ctypes.c_int32), ("row_chunks", ctypes.c_int32),
                ("smem_per_warp", ctypes.c_int32), ("warps_per_block", ctypes.c_int32),
                ("queue_kind", ctypes.c_int32), ("visited_global", ctypes.c_int32)]


_lib = None


def lib():
    """Load libsong.so (raises if it was not built: no fallback exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                              "(there is no CPU fallback for the SONG search)")
        L = ctypes.CDLL(LIB_PATH)
        P, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        PP = ctypes.POINTER(ctypes.c_void_p)
        L.song_default_params.restype = None
        L.song_default_params.argtypes = [ctypes.POINTER(SearchParams), i32, i32]
        L.song_index_create.argtypes = [P, i64, i32, P, i32, i32, PP]
        L.song_index_create_device.argtypes = [P, i64, i32, P, i32, i32, P, PP]
        L.song_index_destroy.argtypes = [P]
        L.song_index_get_info.argtypes = [P, ctypes.POINTER(IndexInfo)]
        L.song_search.argtypes = [P, P, i64, i32, i32, P, P]
        L.song_search_ex.argtypes = [P, ctypes.POINTER(SearchParams), P, i64, P, P, P, P]
        L.song_search_pipelined.argtypes = [P, ctypes.POINTER(SearchParams), P, i64, i64, P, P]
        L.song_index_last_status.argtypes = [P]
        L.song_merge_topk.argtypes = [P, P, i32, i64, i32, i32, P, P, P]
        L.song_rp_encode.argtypes = [P, i64, i32, P, i32, P, P]
        L.song_index_create_codes.argtypes = [P, i64, i32, P, i32, PP]
        L.song_index_create_rp.argtypes = [P, i64, i32, P, i32, P, i32, PP]
        L.song_search_codes_ex.argtypes = [P, ctypes.POINTER(SearchParams), P, i64, P, P, P, P]
        L.song_build_graph.argtypes = [P, i64, i32, i32, i32, P, P]
        L.song_build_graph_batched.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, P, P]
        L.song_build_graph_from_forward.argtypes = [P, i64, i32, i32, i32, P, P, P, P]
        L.song_search_plan_get.argtypes = [ctypes.POINTER(SearchParams), i32, i32,
                                           ctypes.POINTER(SearchPlan)]
        L.song_stage_cycles.argtypes = [P, P, i32]
        L.song_graph_merge_rows.argtypes = [P, P, i64, i32, i32, P, P]
        L.song_merge_topk_peers.argtypes = [P, P, P, i32, i32, i64, i32, i32, ctypes.c_uint32,
                                            P, P, P]
        L.song_last_error.restype = ctypes.c_char_p
        L.song_last_error.argtypes = []
        L.song_version.restype = ctypes.c_char_p
        L.song_version.argtypes = []
        for name in ("song_index_create", "song_index_create_device", "song_index_destroy",
                     "song_index_get_info", "song_search", "song_search_ex",
                     "song_index_last_status", "song_merge_topk", "song_rp_encode",
                     "song_index_create_codes", "song_index_create_rp",
                     "song_search_codes_ex", "song_build_graph", "song_build_graph_batched",
                     "song_build_graph_from_forward", "song_search_plan_get",
                     "song_stage_cycles", "song_merge_topk_peers", "song_graph_merge_rows"):
            getattr(L, name).restype = ctypes.c_int
        _lib = L
    return _lib


def _check(rc: int):
    if rc != 0:
        raise SongError(rc, lib().song_last_error().decode())


def _torch():
    import torch  # plumbing only: device memory + streams
    return torch


def _is_cuda_tensor(x) -> bool:
    try:
        torch = _torch()
    except ImportError:
        return False
    return isinstance(x, torch.Tensor) and x.is_cuda


def _stream_ptr(device) -> ctypes.c_void_p:
    torch = _torch()
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


@dataclass
class Params:
    """song_search_params (include/song.h)."""
    K: int = 10
    queue_len: int = 64
    visited: str = "hash"
    bloom_log2_bits: int = 0
    entry: int = 0
    max_iters: int = 0
    warps_per_block: int = 0
    blocks_per_sm: int = 0
    id_offset: int = 0
    table_log2: int = 0
    steps: int = 1  # multi-step probing (pops per iteration, §V)
    visited_cap: int = 0  # hash deletion schedule: 0 lazy (default cap), >0 lazy cap, -1 eager
    schedule: str = "auto"  # ticket order: "auto" | "batch" | "outlier_first"
    queue_kind: str = "auto"  # "auto" | "separate" (q, topk) | "union" (reading R17)
    queries_per_warp: int = 0  # Fig. 8 packing kernel: 1, 2 or 4 queries per warp (0 = default kernel)

    def to_c(self) -> SearchParams:
        p = SearchParams()
        lib().song_default_params(ctypes.byref(p), self.K, self.queue_len)
        p.visited = VISITED[self.visited]
        p.bloom_log2_bits = self.bloom_log2_bits
        p.entry = self.entry
        p.max_iters = self.max_iters
        p.warps_per_block = self.warps_per_block
        p.blocks_per_sm = self.blocks_per_sm
        p.id_offset = self.id_offset
        p.table_log2 = self.table_log2
        p.steps = self.steps
        p.visited_cap = self.visited_cap
        p.schedule = SCHEDULES[self.schedule]
        p.queue_kind = QUEUE_KINDS[self.queue_kind]
        p.queries_per_warp = self.queries_per_warp
        return p


class SongIndex:
    """song_index_create / song_search / song_index_destroy.

    ``vectors`` [n, dim] float32 and ``adjacency`` [n, degree] int32 may be
    numpy arrays (host create) or CUDA tensors (device create)."""

    def __init__(self, vectors, adjacency, metric: str = "l2", *, _handle=None):
        self._h = ctypes.c_void_p()
        self.metric = metric
        if _handle is not None:  # made by from_codes / from_rp
            self._h = _handle
            self.device = None
            info = self.info()
            self.n, self.dim, self.degree = info.n, info.dim, info.degree
            self.code_bits = info.code_bits
            return
        m = METRICS[metric]
        self.code_bits = 0
        if _is_cuda_tensor(vectors):
            torch = _torch()
            v = vectors.contiguous().to(torch.float32)
            a = adjacency.to(device=v.device, dtype=torch.int32).contiguous()
            self.device = v.device
            with torch.cuda.device(v.device):
                _check(lib().song_index_create_device(
                    ctypes.c_void_p(v.data_ptr()), v.shape[0], v.shape[1],
                    ctypes.c_void_p(a.data_ptr()), a.shape[1], m, _stream_ptr(v.device),
                    ctypes.byref(self._h)))
        else:
            v = np.ascontiguousarray(vectors, np.float32)
            a = np.ascontiguousarray(adjacency, np.int32)
            assert v.ndim == 2 and a.ndim == 2 and a.shape[0] == v.shape[0]
            self.device = None
            _check(lib().song_index_create(
                v.ctypes.data_as(ctypes.c_void_p), v.shape[0], v.shape[1],
                a.ctypes.data_as(ctypes.c_void_p), a.shape[1], m, ctypes.byref(self._h)))
        info = self.info()
        self.n, self.dim, self.degree = info.n, info.dim, info.degree

    @classmethod
    def from_codes(cls, codes: np.ndarray, bits: int, adjacency) -> "SongIndex":
        """song_index_create_codes: HOST codes [n, bits/32] uint32 (§VII)."""
        c = np.ascontiguousarray(codes, np.uint32)
        a = np.ascontiguousarray(adjacency, np.int32)
        h = ctypes.c_void_p()
        _check(lib().song_index_create_codes(c.ctypes.data_as(ctypes.c_void_p), c.shape[0], bits,
                                             a.ctypes.data_as(ctypes.c_void_p), a.shape[1],
                                             ctypes.byref(h)))
        return cls(None, None, "hamming", _handle=h)

    @classmethod
    def from_rp(cls, vectors: np.ndarray, R: np.ndarray, adjacency) -> "SongIndex":
        """song_index_create_rp: HOST vectors [n, dim] streamed to the device and
        encoded with HOST R [bits, dim]; only the codes stay resident."""
        v = np.ascontiguousarray(vectors, np.float32)
        r = np.ascontiguousarray(R, np.float32)
        a = np.ascontiguousarray(adjacency, np.int32)
        assert r.shape[1] == v.shape[1]
        h = ctypes.c_void_p()
        _check(lib().song_index_create_rp(v.ctypes.data_as(ctypes.c_void_p), v.shape[0],
                                          v.shape[1], r.ctypes.data_as(ctypes.c_void_p),
                                          r.shape[0], a.ctypes.data_as(ctypes.c_void_p),
                                          a.shape[1], ctypes.byref(h)))
        return cls(None, None, "hamming", _handle=h)

    def search_codes(self, qcodes, params: "Params", counters: bool = False):
        """song_search_codes_ex on CUDA uint32/int32 code tensors [nq, bits/32]."""
        torch = _torch()
        if not _is_cuda_tensor(qcodes):
            raise TypeError("search_codes() takes a CUDA tensor")
        q = qcodes.contiguous()
        assert q.element_size() == 4
        nq = q.shape[0]
        ids = torch.empty((nq, params.K), dtype=torch.int32, device=q.device)
        dists = torch.empty((nq, params.K), dtype=torch.float32, device=q.device)
        ctr = torch.empty((nq, 2), dtype=torch.int32, device=q.device) if counters else None
        cp = params.to_c()
        _check(lib().song_search_codes_ex(
            self._h, ctypes.byref(cp), ctypes.c_void_p(q.data_ptr()), nq,
            ctypes.c_void_p(ids.data_ptr()), ctypes.c_void_p(dists.data_ptr()),
            ctypes.c_void_p(ctr.data_ptr() if ctr is not None else 0), _stream_ptr(q.device)))
        return (ids, dists, ctr) if counters else (ids, dists)

    def info(self) -> IndexInfo:
        inf = IndexInfo()
        _check(lib().song_index_get_info(self._h, ctypes.byref(inf)))
        return inf

    def search_host(self, queries: np.ndarray, K: int, queue_len: int) -> Tuple[np.ndarray, np.ndarray]:
        """song_search: HOST buffers in and out (HtoD + kernel + DtoH inside)."""
        q = np.ascontiguousarray(queries, np.float32)
        if q.ndim == 1:
            q = q[None]
        ids = np.empty((q.shape[0], K), np.int32)
        dists = np.empty((q.shape[0], K), np.float32)
        self.search_host_into(q, K, queue_len, ids, dists)
        return ids, dists

    def search_host_into(self, q, K, queue_len, ids, dists):
        """song_search into caller buffers (numpy or pinned CPU tensors)."""
        def ptr(x):
            return ctypes.c_void_p(x.data_ptr() if hasattr(x, "data_ptr") else
                                   x.ctypes.data)
        _check(lib().song_search(self._h, ptr(q), q.shape[0], K, queue_len, ptr(ids), ptr(dists)))

    def search_pipelined_into(self, q, params: "Params", ids, dists):
        """song_search_pipelined: q [nbatch, nq, dim] HOST (numpy or pinned CPU
        tensor), ids / dists [nbatch, nq, K] HOST; blocking."""
        def ptr(x):
            return ctypes.c_void_p(x.data_ptr() if hasattr(x, "data_ptr") else
                                   x.ctypes.data)
        if len(q.shape) != 3 or tuple(ids.shape) != (q.shape[0], q.shape[1], params.K) \
                or tuple(dists.shape) != tuple(ids.shape):
            raise ValueError("q [nbatch, nq, dim], ids / dists [nbatch, nq, K]")
        pc = params.to_c()
        _check(lib().song_search_pipelined(self._h, ctypes.byref(pc), ptr(q), q.shape[0],
                                           q.shape[1], ptr(ids), ptr(dists)))

    def search_pipelined(self, queries: np.ndarray, params: "Params"):
        """song_search_pipelined on host batches [nbatch, nq, dim] -> (ids, dists)."""
        q = np.ascontiguousarray(queries, np.float32)
        ids = np.empty((q.shape[0], q.shape[1], params.K), np.int32)
        dists = np.empty(ids.shape, np.float32)
        self.search_pipelined_into(q, params, ids, dists)
        return ids, dists

    def search(self, queries, K: int = 10, queue_len: int = 64, params: Optional[Params] = None,
               counters: bool = False, out=None):
        """song_search_ex on CUDA tensors (async on torch's current stream).
        Returns (ids [nq,K] int32, dists [nq,K] f32[, counters [nq,2] int32])."""
        torch = _torch()
        if not _is_cuda_tensor(queries):
            raise TypeError("search() takes a CUDA tensor; use search_host() for host arrays")
        p = params or Params(K=K, queue_len=queue_len)
        q = queries.contiguous()
        if q.dtype != torch.float32:
            q = q.float()
        nq = q.shape[0]
        if out is None:
            ids = torch.empty((nq, p.K), dtype=torch.int32, device=q.device)
            dists = torch.empty((nq, p.K), dtype=torch.float32, device=q.device)
            ctr = torch.empty((nq, 2), dtype=torch.int32, device=q.device) if counters else None
        else:
            ids, dists, ctr = out
        cp = p.to_c()
        _check(lib().song_search_ex(
            self._h, ctypes.byref(cp), ctypes.c_void_p(q.data_ptr()), nq,
            ctypes.c_void_p(ids.data_ptr()), ctypes.c_void_p(dists.data_ptr()),
            ctypes.c_void_p(ctr.data_ptr() if ctr is not None else 0), _stream_ptr(q.device)))
        return (ids, dists, ctr) if counters else (ids, dists)

    def plan(self, params: "Params") -> "SearchPlan":
        """song_search_plan_get for this index (its dimension and metric)."""
        info = self.info()
        dim = info.dim_padded if self.metric == "hamming" else info.dim
        return plan(params, dim, self.metric)

    def stage_cycles(self, reset: bool = True):
        """song_stage_cycles (SONG_STAGE_TIMING builds): SM cycles per stage
        [pop/topk, locate, distance, maintenance] summed over warps."""
        out = np.zeros(4, np.uint64)
        _check(lib().song_stage_cycles(self._h, out.ctypes.data_as(ctypes.c_void_p), int(reset)))
        return out

    def last_status(self):
        """Synchronise and raise SongError if a query was flagged."""
        _check(lib().song_index_last_status(self._h))

    def close(self):
        if self._h:
            lib().song_index_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def merge_topk(ids, dists, K: int):
    """song_merge_topk: ids/dists [G, nq, Kin] CUDA tensors (rows sorted by
    (dist, id), global ids) -> the K best per query [nq, K]."""
    torch = _torch()
    ids = ids.to(torch.int32).contiguous()
    dists = dists.to(torch.float32).contiguous()
    G, nq, kin = ids.shape
    oi = torch.empty((nq, K), dtype=torch.int32, device=ids.device)
    od = torch.empty((nq, K), dtype=torch.float32, device=ids.device)
    _check(lib().song_merge_topk(ctypes.c_void_p(ids.data_ptr()), ctypes.c_void_p(dists.data_ptr()),
                                 G, nq, kin, K, ctypes.c_void_p(oi.data_ptr()),
                                 ctypes.c_void_p(od.data_ptr()), _stream_ptr(ids.device)))
    return oi, od


def merge_graph_rows(first, second, take_first: int):
    """song_graph_merge_rows (reading R18): CUDA int32 [n, degree] graphs ->
    the merged rows (first `take_first` of `first`, then `second`, then the
    rest of `first`; ids once, -1 padded)."""
    torch = _torch()
    a = first.to(torch.int32).contiguous()
    b = second.to(device=a.device, dtype=torch.int32).contiguous()
    assert a.shape == b.shape
    out = torch.empty_like(a)
    _check(lib().song_graph_merge_rows(ctypes.c_void_p(a.data_ptr()), ctypes.c_void_p(b.data_ptr()),
                                       a.shape[0], a.shape[1], int(take_first),
                                       ctypes.c_void_p(out.data_ptr()), _stream_ptr(a.device)))
    return out


def build_graph_mips(vectors, degree: int = 32, take_ip: int = 8, prefix: int = 1 << 16,
                     queue_len: int = 128, batch_shift: int = 2):
    """Reading R18: the inner-product graph = each vertex's first `take_ip`
    links of the IP graph (song_build_graph, exact insertion) filled with the
    angular graph's (song_build_graph_batched, cosine)."""
    ip = build_graph(vectors, degree, "ip")
    cos = build_graph_batched(vectors, degree, "cosine", prefix=prefix, queue_len=queue_len,
                              batch_shift=batch_shift)
    return merge_graph_rows(ip, cos, take_ip)


def merge_topk_peers(ids_ptrs, dists_ptrs, nq: int, kin: int, K: int, out=None,
                     sig_ptrs=None, rank: int = 0, epoch: int = 0, device=None):
    """song_merge_topk_peers: ``ids_ptrs`` / ``dists_ptrs`` are CUDA int64
    tensors [G] holding the device addresses of each rank's [nq, kin] rows
    (peer-mapped, e.g. symmetric memory); ``sig_ptrs`` the [G] signal-pad
    addresses or None.  Returns (ids [nq, K], dists [nq, K]) on ``device``."""
    torch = _torch()
    dev = device or ids_ptrs.device
    G = int(ids_ptrs.numel())
    if out is None:
        oi = torch.empty((nq, K), dtype=torch.int32, device=dev)
        od = torch.empty((nq, K), dtype=torch.float32, device=dev)
    else:
        oi, od = out
    _check(lib().song_merge_topk_peers(
        ctypes.c_void_p(ids_ptrs.data_ptr()), ctypes.c_void_p(dists_ptrs.data_ptr()),
        ctypes.c_void_p(sig_ptrs.data_ptr() if sig_ptrs is not None else 0), int(rank), G,
        int(nq), int(kin), int(K), int(epoch), ctypes.c_void_p(oi.data_ptr()),
        ctypes.c_void_p(od.data_ptr()), _stream_ptr(dev)))
    return oi, od


def build_graph(vectors, degree: int = 32, metric: str = "l2"):
    """song_build_graph: CUDA tensor vectors [n, dim] -> adjacency [n, degree]
    int32 CUDA tensor (NSW forward lists + backward lists + HNSW heuristic,
    DESIGN.md reading R15)."""
    torch = _torch()
    if not _is_cuda_tensor(vectors):
        raise TypeError("build_graph() takes a CUDA tensor")
    v = vectors.contiguous().float()
    adj = torch.empty((v.shape[0], degree), dtype=torch.int32, device=v.device)
    with torch.cuda.device(v.device):
        _check(lib().song_build_graph(ctypes.c_void_p(v.data_ptr()), v.shape[0], v.shape[1],
                                      METRICS[metric], degree, ctypes.c_void_p(adj.data_ptr()),
                                      _stream_ptr(v.device)))
    return adj


def build_graph_batched(vectors, degree: int = 32, metric: str = "l2", prefix: int = 1 << 20,
                        queue_len: int = 64, batch_shift: int = 1):
    """song_build_graph_batched (reading R16, the scale-out builder):
    exact forward lists for the first `prefix` rows, then batches of
    max(1, m >> batch_shift) rows search the graph of the rows before them
    (K = degree, `queue_len`) for their forward lists."""
    torch = _torch()
    if not _is_cuda_tensor(vectors):
        raise TypeError("build_graph_batched() takes a CUDA tensor")
    v = vectors.contiguous().float()
    adj = torch.empty((v.shape[0], degree), dtype=torch.int32, device=v.device)
    with torch.cuda.device(v.device):
        _check(lib().song_build_graph_batched(
            ctypes.c_void_p(v.data_ptr()), v.shape[0], v.shape[1], METRICS[metric], degree,
            int(prefix), int(queue_len), int(batch_shift), ctypes.c_void_p(adj.data_ptr()),
            _stream_ptr(v.device)))
    return adj


def build_graph_from_forward(vectors, fwd_ids, fwd_dists, metric: str = "l2"):
    """song_build_graph_from_forward: R15 steps 2-4 on given forward lists
    (CUDA tensors [n, degree], rows ascending by (dist, id), -1 padded)."""
    torch = _torch()
    v = vectors.contiguous().float()
    fi = fwd_ids.to(torch.int32).contiguous()
    fd = fwd_dists.to(torch.float32).contiguous()
    adj = torch.empty(fi.shape, dtype=torch.int32, device=v.device)
    with torch.cuda.device(v.device):
        _check(lib().song_build_graph_from_forward(
            ctypes.c_void_p(v.data_ptr()), v.shape[0], v.shape[1], METRICS[metric], fi.shape[1],
            ctypes.c_void_p(fi.data_ptr()), ctypes.c_void_p(fd.data_ptr()),
            ctypes.c_void_p(adj.data_ptr()), _stream_ptr(v.device)))
    return adj


def plan(params: "Params", dim: int, metric: str = "l2") -> SearchPlan:
    """song_search_plan_get: the resolved sizes and launch shape of a search
    (host-only, no GPU needed).  ``dim`` is the index dimension (code words
    for "hamming")."""
    out = SearchPlan()
    cp = params.to_c()
    _check(lib().song_search_plan_get(ctypes.byref(cp), int(dim), METRICS[metric],
                                      ctypes.byref(out)))
    return out


def default_visited_cap(L: int, dim: int = 128, metric: str = "l2", K: int = 1) -> int:
    """The lazy-deletion capacity C the library uses for visited_cap = 0
    (read from song_search_plan_get, the single source of the default)."""
    return int(plan(Params(K=min(K, L), queue_len=L), dim, metric).visited_cap)


def rp_encode(vectors, R):
    """song_rp_encode: CUDA tensors vectors [n, dim], R [bits, dim] fp32 ->
    codes [n, bits/32] (int32 tensor holding the uint32 words, §VII)."""
    torch = _torch()
    v = vectors.contiguous().float()
    r = R.to(device=v.device, dtype=torch.float32).contiguous()
    bits = r.shape[0]
    codes = torch.empty((v.shape[0], bits // 32 if bits % 32 == 0 else 1), dtype=torch.int32,
                        device=v.device)
    _check(lib().song_rp_encode(ctypes.c_void_p(v.data_ptr()), v.shape[0], v.shape[1],
                                ctypes.c_void_p(r.data_ptr()), bits,
                                ctypes.c_void_p(codes.data_ptr()), _stream_ptr(v.device)))
    return codes


def version() -> str:
    return lib().song_version().decode()
