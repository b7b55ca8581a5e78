"""Multi-GPU orchestration over torch.distributed (one process per GPU).

Two modes:

* **query sharding** — every rank holds a replica of the index and searches its
  own slice of the batch; the search has no data-path collective ("SONG
  can also linearly scale with multiple GPU cards").  Results may optionally be
  gathered to every rank.
* **dataset sharding** — P:471: "shard the data for each GPU, build a graph
  index for each shard, perform graph search on each GPU and merge the
  results".  Rank r owns ids [lo_r, hi_r) with its own graph; the queries are
  broadcast, each rank searches its shard returning global ids (search
  parameter ``id_offset``).  On NCCL (one node) the search writes straight
  into symmetric-memory buffers and ONE kernel per rank
  (``song_merge_topk_peers``, :class:`PeerMerger`) signals the peers through
  their signal pads and merges straight from their buffers over NVLink — the
  gather is the merge's own loads.  Elsewhere (gloo tests) the per-rank
  lists are all-gathered and merged by ``song_merge_topk``.

The search and merge steps are injectable so the host logic can be tested with
the gloo backend on CPU (tests/test_sharded_gloo.py); the product defaults are
the CUDA kernels behind libsong.so.
"""
from __future__ import annotations

from typing import Callable, List, Optional, Tuple

import torch
import torch.distributed as dist


def shard_ranges(n: int, world: int) -> List[Tuple[int, int]]:
    """Contiguous, balanced id ranges [lo, hi) for each rank."""
    base, extra = divmod(n, world)
    out, lo = [], 0
    for r in range(world):
        hi = lo + base + (1 if r < extra else 0)
        out.append((lo, hi))
        lo = hi
    return out


def query_slice(nq: int, rank: int, world: int) -> Tuple[int, int]:
    return shard_ranges(nq, world)[rank]


def _default_searcher(index, params):
    def run(queries: torch.Tensor, id_offset: int):
        from .song import Params
        p = Params(**{**params.__dict__, "id_offset": id_offset})
        return index.search(queries, params=p)
    return run


def _default_merger(K: int):
    def run(ids: torch.Tensor, dists: torch.Tensor):
        from .song import merge_topk
        return merge_topk(ids, dists, K)
    return run


def query_sharded_search(searcher: Callable, queries_local: torch.Tensor,
                         gather: bool = False, group=None):
    """Search this rank's queries; optionally all-gather [nq, K] results."""
    ids, dists = searcher(queries_local, 0)
    if not gather or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return ids, dists
    world = dist.get_world_size(group)
    sizes = [torch.zeros(1, dtype=torch.int64, device=ids.device) for _ in range(world)]
    dist.all_gather(sizes, torch.tensor([ids.shape[0]], dtype=torch.int64, device=ids.device),
                    group=group)
    mx = int(max(s.item() for s in sizes))
    pad_i = torch.full((mx, ids.shape[1]), -1, dtype=ids.dtype, device=ids.device)
    pad_d = torch.full((mx, dists.shape[1]), float("inf"), dtype=dists.dtype, device=ids.device)
    pad_i[:ids.shape[0]] = ids
    pad_d[:dists.shape[0]] = dists
    gi = [torch.empty_like(pad_i) for _ in range(world)]
    gd = [torch.empty_like(pad_d) for _ in range(world)]
    dist.all_gather(gi, pad_i, group=group)
    dist.all_gather(gd, pad_d, group=group)
    ids = torch.cat([g[:int(s.item())] for g, s in zip(gi, sizes)])
    dists = torch.cat([g[:int(s.item())] for g, s in zip(gd, sizes)])
    return ids, dists


def dataset_sharded_search(searcher: Callable, merger: Callable, queries: Optional[torch.Tensor],
                           nq: int, dim: int, K: int, id_offset: int, device,
                           group=None, src: int = 0):
    """P:471 over `group`: broadcast the queries from `src`, search the local
    shard (ids offset to global), all-gather the [nq, K] lists, merge.

    Returns the merged (ids [nq, K] int32, dists [nq, K] f32) on every rank."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    if rank == src:
        q = queries.to(device=device, dtype=torch.float32).contiguous()
    else:
        q = torch.empty((nq, dim), dtype=torch.float32, device=device)
    if world > 1:
        dist.broadcast(q, src=src, group=group)
    ids, dists = searcher(q, id_offset)
    ids = ids.to(torch.int32).contiguous()
    dists = dists.to(torch.float32).contiguous()
    if world > 1:
        gi = torch.empty((world,) + tuple(ids.shape), dtype=torch.int32, device=ids.device)
        gd = torch.empty((world,) + tuple(dists.shape), dtype=torch.float32, device=ids.device)
        if dist.get_backend(group) == "nccl":
            dist.all_gather_into_tensor(gi, ids, group=group)
            dist.all_gather_into_tensor(gd, dists, group=group)
        else:
            dist.all_gather(list(gi.unbind(0)), ids, group=group)
            dist.all_gather(list(gd.unbind(0)), dists, group=group)
    else:
        gi, gd = ids[None], dists[None]
    return merger(gi, gd)


class PeerMerger:
    """Fused gather + merge over torch symmetric memory (NCCL group, one
    node): [nq, kin] ids / dists buffers every rank can address, a private
    signal pad per rank, and the epoch of the next merge."""

    def __init__(self, nq: int, kin: int, K: int, device, group=None):
        import torch.distributed._symmetric_memory as symm_mem
        grp = group or dist.group.WORLD
        self.G, self.rank = dist.get_world_size(grp), dist.get_rank(grp)
        self.nq, self.kin, self.K, self.device = nq, kin, K, device
        name = grp.group_name
        try:
            symm_mem.enable_symm_mem_for_group(name)
        except Exception:  # newer torch: always enabled
            pass
        self.ids = symm_mem.empty((nq, kin), dtype=torch.int32, device=device)
        self.dists = symm_mem.empty((nq, kin), dtype=torch.float32, device=device)
        self.sig = symm_mem.empty((max(self.G, 1),), dtype=torch.int32, device=device)
        self.sig.zero_()
        hs = [symm_mem.rendezvous(t, name) for t in (self.ids, self.dists, self.sig)]
        ptrs = lambda h: torch.tensor([int(p) for p in h.buffer_ptrs], dtype=torch.int64,  # noqa: E731
                                      device=device)
        self.ids_ptrs, self.dists_ptrs, self.sig_ptrs = (ptrs(h) for h in hs)
        self._handles = hs
        torch.cuda.synchronize(device)
        dist.barrier(grp)  # every pad is zero before the first merge
        self.epoch = 0

    def merge(self, out=None):
        """song_merge_topk_peers on this rank's stream (after its search
        wrote self.ids / self.dists): returns (ids [nq, K], dists [nq, K])."""
        from .song import merge_topk_peers
        self.epoch += 1
        return merge_topk_peers(self.ids_ptrs, self.dists_ptrs, self.nq, self.kin, self.K,
                                out=out, sig_ptrs=self.sig_ptrs, rank=self.rank,
                                epoch=self.epoch, device=self.device)


def dataset_sharded_search_fused(index, params, merger: PeerMerger, queries: Optional[torch.Tensor],
                                 nq: int, dim: int, id_offset: int, device, group=None,
                                 src: int = 0, out=None):
    """P:471 with the fused gather + merge: broadcast the queries, search the
    local shard into the symmetric buffers, merge from every peer's buffers."""
    from .song import Params
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    if rank == src:
        q = queries.to(device=device, dtype=torch.float32).contiguous()
    else:
        q = torch.empty((nq, dim), dtype=torch.float32, device=device)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.broadcast(q, src=src, group=group)
    p = Params(**{**params.__dict__, "id_offset": id_offset})
    index.search(q, params=p, out=(merger.ids, merger.dists, None))
    return merger.merge(out=out)


class ShardedIndex:
    """Dataset-sharded SONG index: this rank's shard of the vectors with its
    own graph, searched with global ids and merged across ranks."""

    def __init__(self, vectors_shard, adjacency_shard, id_offset: int, metric: str = "l2",
                 group=None):
        from .song import SongIndex
        self.index = SongIndex(vectors_shard, adjacency_shard, metric=metric)
        self.id_offset = id_offset
        self.group = group
        self.dim = self.index.dim

    def search(self, queries: Optional[torch.Tensor], nq: int, K: int, queue_len: int,
               fused: bool = True, **params):
        """Search every rank's shard and merge; ``fused`` (NCCL) merges over
        symmetric memory in one kernel, else NCCL all-gather + merge kernel."""
        from .song import Params
        p = Params(K=K, queue_len=queue_len, **params)
        dev = torch.device("cuda", torch.cuda.current_device())
        if fused and dist.is_initialized() and dist.get_backend(self.group) == "nccl":
            m = getattr(self, "_merger", None)
            if m is None or (m.nq, m.kin, m.K) != (nq, K, K):
                m = self._merger = PeerMerger(nq, K, K, dev, group=self.group)
            return dataset_sharded_search_fused(self.index, p, m, queries, nq, self.dim,
                                                self.id_offset, dev, group=self.group)
        return dataset_sharded_search(_default_searcher(self.index, p), _default_merger(K),
                                      queries, nq, self.dim, K, self.id_offset, dev,
                                      group=self.group)
