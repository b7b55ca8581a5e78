"""Proximity-graph construction (tooling; SONG itself loads pre-built graphs,
P:477).

``build_graph`` makes a fixed-degree, HNSW-layer-0-style graph:

1. *exact-insertion NSW* [46]: vertex i links to its M nearest among the
   vertices inserted before it (ids 0..i-1), found exactly (blocked GEMM +
   top-k).  Early vertices therefore carry the long-range links that make the
   fixed entry vertex 0 a good "default starting point".
2. reverse edges (NSW links are bidirectional), capped at the R nearest;
3. the HNSW neighbour-selection heuristic prunes each candidate list to
   ``degree``; free slots are refilled with the nearest pruned candidates and
   the rest padded with -1 (fixed-degree rows).

Runs with torch on any device; deterministic on CPU (the tiny config) and on
the GPU up to the tie order of torch.topk.  Distances here are graph-building
heuristics only — never the search's arithmetic.
"""
from __future__ import annotations

import torch


def _pair_dist(a: torch.Tensor, b: torch.Tensor, metric: str, bn2=None) -> torch.Tensor:
    if metric == "l2":
        an2 = (a * a).sum(1, keepdim=True)
        bn2 = (b * b).sum(1) if bn2 is None else bn2
        return (an2 + bn2[None, :] - 2.0 * (a @ b.T)).clamp_min_(0)
    return -(a @ b.T)  # ip; cosine inputs arrive normalised


def _prefix_knn(x: torch.Tensor, M: int, metric: str, row_block: int, col_block: int):
    """For every i: the M nearest j < i (padded with -1 / inf)."""
    n = x.shape[0]
    dev = x.device
    ids = torch.full((n, M), -1, dtype=torch.int64, device=dev)
    dst = torch.full((n, M), float("inf"), device=dev)
    xn2 = (x * x).sum(1) if metric == "l2" else None
    for r0 in range(0, n, row_block):
        r1 = min(n, r0 + row_block)
        rows = x[r0:r1]
        best_d = torch.full((r1 - r0, M), float("inf"), device=dev)
        best_i = torch.full((r1 - r0, M), -1, dtype=torch.int64, device=dev)
        ri = torch.arange(r0, r1, device=dev)[:, None]
        for c0 in range(0, r1 - 1 if r1 > 1 else 0, col_block):
            c1 = min(r1, c0 + col_block)
            d = _pair_dist(rows, x[c0:c1], metric, None if xn2 is None else xn2[c0:c1])
            cj = torch.arange(c0, c1, device=dev)[None, :]
            d = d.masked_fill(cj >= ri, float("inf"))
            k = min(M, c1 - c0)
            td, ti = torch.topk(d, k, dim=1, largest=False)
            cat_d = torch.cat([best_d, td], 1)
            cat_i = torch.cat([best_i, ti + c0], 1)
            sd, si = torch.topk(cat_d, M, dim=1, largest=False)
            best_d = sd
            best_i = torch.gather(cat_i, 1, si)
        best_i = torch.where(torch.isinf(best_d), torch.full_like(best_i, -1), best_i)
        ids[r0:r1] = best_i
        dst[r0:r1] = best_d
    return ids, dst


def _heuristic_prune(x, cand, cand_d, degree, metric, block):
    """HNSW's neighbour heuristic: walk candidates nearest-first, keep c if it
    is closer to the base vertex than to every kept neighbour; then refill."""
    n, C = cand.shape
    out = torch.full((n, degree), -1, dtype=torch.int64, device=x.device)
    for r0 in range(0, n, block):
        r1 = min(n, r0 + block)
        ci = cand[r0:r1]
        cd = cand_d[r0:r1]
        valid = ci >= 0
        vec = x[ci.clamp_min(0)]                       # [b, C, dim]
        if metric == "l2":
            nn = (vec * vec).sum(-1)
            pd = (nn[:, :, None] + nn[:, None, :] - 2 * torch.bmm(vec, vec.transpose(1, 2))).clamp_min(0)
        else:
            pd = -torch.bmm(vec, vec.transpose(1, 2))
        keep = torch.zeros_like(valid)
        nkeep = torch.zeros(r1 - r0, dtype=torch.int64, device=x.device)
        big = torch.finfo(pd.dtype).max
        for t in range(C):
            # min distance from candidate t to already-kept candidates
            m = torch.where(keep, pd[:, t, :], torch.full_like(pd[:, t, :], big)).min(1).values
            ok = valid[:, t] & (m > cd[:, t]) & (nkeep < degree)
            keep[:, t] = ok
            nkeep += ok.long()
        # refill with the nearest pruned candidates (keepPrunedConnections)
        rank_keep = torch.where(keep, torch.zeros_like(cd), torch.ones_like(cd))
        order_key = rank_keep * 1e30 + torch.where(valid, cd, torch.full_like(cd, 1e38))
        order_key = torch.where(valid, order_key, torch.full_like(cd, float("inf")))
        # stable order: kept (in distance order) first, then pruned by distance
        srt = torch.sort(order_key, dim=1, stable=True).indices[:, :degree]
        sel = torch.gather(ci, 1, srt)
        sel_valid = torch.gather(valid, 1, srt)
        out[r0:r1, :srt.shape[1]] = torch.where(sel_valid, sel, torch.full_like(sel, -1))
    return out


def build_graph(x: torch.Tensor, degree: int = 32, metric: str = "l2", M: int = None,
                rev_cap: int = None, row_block: int = 8192, col_block: int = 65536,
                prune_block: int = 8192, heuristic: bool = True) -> torch.Tensor:
    """Returns int32 adjacency [n, degree] (-1 padded) on x's device.
    heuristic=False keeps the `degree` nearest of F(v) u B(v) (plain NSW lists,
    probe only: reading R15 always applies the heuristic)."""
    x = x.float()
    if metric == "cosine":
        x = x / x.norm(dim=1, keepdim=True).clamp_min(1e-30)
    n = x.shape[0]
    M = M or degree
    rev_cap = rev_cap or degree
    fwd, fwd_d = _prefix_knn(x, M, metric, row_block, col_block)
    # reverse edges: j <- i for every forward edge i -> j; keep the rev_cap nearest
    src = torch.arange(n, device=x.device)[:, None].expand(n, M).reshape(-1)
    dstv = fwd.reshape(-1)
    dd = fwd_d.reshape(-1)
    ok = dstv >= 0
    src, dstv, dd = src[ok], dstv[ok], dd[ok]
    # sort by (dst, dist) and take the first rev_cap per dst
    order = torch.argsort(dd, stable=True)
    src, dstv, dd = src[order], dstv[order], dd[order]
    order = torch.argsort(dstv, stable=True)
    src, dstv, dd = src[order], dstv[order], dd[order]
    counts = torch.bincount(dstv, minlength=n)
    starts = torch.cumsum(counts, 0) - counts
    rank = torch.arange(dstv.shape[0], device=x.device) - starts[dstv]
    keep = rank < rev_cap
    rev = torch.full((n, rev_cap), -1, dtype=torch.int64, device=x.device)
    rev_d = torch.full((n, rev_cap), float("inf"), device=x.device)
    rev[dstv[keep], rank[keep]] = src[keep]
    rev_d[dstv[keep], rank[keep]] = dd[keep]
    cand = torch.cat([fwd, rev], 1)
    cand_d = torch.cat([fwd_d, rev_d], 1)
    cand_d = torch.where(cand >= 0, cand_d, torch.full_like(cand_d, float("inf")))
    srt = torch.sort(cand_d, dim=1, stable=True).indices
    cand = torch.gather(cand, 1, srt)
    cand_d = torch.gather(cand_d, 1, srt)
    if not heuristic:
        return cand[:, :degree].to(torch.int32)
    adj = _heuristic_prune(x, cand, cand_d, degree, metric, prune_block)
    return adj.to(torch.int32)
