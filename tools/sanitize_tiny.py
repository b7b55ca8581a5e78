"""Small invocations of every kernel family for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck):

    compute-sanitizer --tool racecheck python tools/sanitize_tiny.py

tiny-config search through every visited kind and queue kind (separate
register or shared-memory q / topk, the bounded union in registers or tiers),
multi-step probing, the pipelined host-buffer path,
Hamming codes, the three graph builders, both merges.  Exits non-zero if a
result disagrees with the oracle on the integer-valued sample."""
from __future__ import annotations

import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def main():
    import numpy as np
    import torch
    import oracle
    from paper_conf_icde_zhaotl20_b200 import song
    from test_gpu_parity import oracle_kw

    rng = np.random.default_rng(3)
    n, dim = 3000, 16
    x = rng.integers(0, 30, (n, dim)).astype(np.float32)
    q = rng.integers(0, 30, (40, dim)).astype(np.float32)
    xt = torch.as_tensor(x, device="cuda")
    adj = song.build_graph(xt, 16)                                   # R15
    adj_b = song.build_graph_batched(xt, 16, prefix=500, queue_len=32)  # R16
    big = torch.where(adj_b >= 0, adj_b, n)
    fi = torch.sort(big, dim=1).values          # (dist 0, id) keys ascending
    fi = torch.where(fi < n, fi, -1).to(torch.int32)
    song.build_graph_from_forward(xt, fi, torch.zeros(fi.shape, device="cuda"))
    idx = song.SongIndex(xt, adj)
    an = adj.cpu().numpy()
    qt = torch.as_tensor(q, device="cuda")
    bad = 0
    cases = [("hash", 24, {}), ("hash", 100, {}), ("hash", 200, {}),
             ("hash", 200, {"queue_kind": "separate"}), ("hash", 40, {"queue_kind": "union"}),
             ("hash", 24, {"queue_kind": "separate"}), ("hash", 100, {"queue_kind": "separate"}),
             ("hash", 100, {"visited_cap": -1}),
             ("hash", 64, {"visited_cap": -1}), ("bloom", 48, {}), ("hashtable", 48, {}),
             ("hashtable-sel", 200, {}), ("cuckoo", 48, {}), ("cuckoo", 200, {}),
             ("hash", 48, {"steps": 2})]
    for visited, L, kw in cases:
        p = song.Params(K=10, queue_len=L, visited=visited, **kw)
        ids, d, c = idx.search(qt, params=p, counters=True)
        torch.cuda.synchronize()
        idx.last_status()
        o = oracle.search(x, an, q, 10, L, **oracle_kw(visited, L, kw.get("steps", 1),
                                                        kw.get("visited_cap", 0), 0,
                                                        kw.get("queue_kind", "auto")))
        ok = (ids.cpu().numpy() == o[0]).all() and (c.cpu().numpy() == o[2]).all()
        print(visited, L, kw, "ok" if ok else "MISMATCH", flush=True)
        bad += not ok
    # Hamming codes
    R = torch.randn(64, dim, device="cuda")
    codes = song.rp_encode(xt, R)
    cidx = song.SongIndex.from_codes(codes.cpu().numpy().view(np.uint32), 64, an)
    cidx.search_codes(song.rp_encode(qt, R), song.Params(K=5, queue_len=32))
    # merges
    ids, d = idx.search(qt, params=song.Params(K=10, queue_len=32))
    mi, md = song.merge_topk(torch.stack([ids, ids + n]), torch.stack([d, d]), 10)
    ids2 = torch.where(ids >= 0, ids + n, -1)
    ptr = torch.tensor([ids.data_ptr(), ids2.data_ptr()], dtype=torch.int64, device="cuda")
    dptr = torch.tensor([d.data_ptr(), d.data_ptr()], dtype=torch.int64, device="cuda")
    song.merge_topk_peers(ptr, dptr, q.shape[0], 10, 10)
    # the pipelined host-buffer path: two lanes, copy streams, concurrent grids
    pp = song.Params(K=10, queue_len=24)
    qb = np.ascontiguousarray(np.stack([q, q[::-1], q]))
    pi, pd = idx.search_pipelined(qb, pp)
    ref = idx.search(qt, params=pp)[0].cpu().numpy()
    ok = (pi[0] == ref).all() and (pi[1] == ref[::-1]).all() and (pi[2] == ref).all()
    print("pipelined", "ok" if ok else "MISMATCH", flush=True)
    bad += not ok
    torch.cuda.synchronize()
    print("sanitize_tiny done,", bad, "mismatches", flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
