"""Would a refinement pass improve the R16 graph?  After the batched build,
every row searches the finished graph (K = 2 D + 1, L = --L) and new forward
lists are taken from the results — all ids except the row itself
("unrestricted") or only earlier ids ("earlier", the NSW rule) — then R15 steps
2-4 rebuild the graph (song_build_graph_from_forward).  Prints recall@10 of the
search on each graph at a few queue lengths.

    python tools/refine_probe.py [--config sift1m]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sift1m")
    ap.add_argument("--L", type=int, default=64)
    ap.add_argument("--out", default="gpurun_out/refine_probe.json")
    a = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS, make_data
    cfg = CONFIGS[a.config]
    x, q = make_data(cfg, device="cuda")
    truth = bench.ground_truth(x, q, 10, cfg.metric)
    D = cfg.degree
    res = {}

    def sweep(adj, name):
        idx = song.SongIndex(x, adj, metric=cfg.metric)
        r = {}
        for L in (16, 20, 24, 32):
            ids, _ = idx.search(q, params=song.Params(K=10, queue_len=L))
            r[L] = round(bench.recall_t(ids, truth), 4)
        idx.close()
        res[name] = r
        print(name, r, flush=True)

    g0 = bench.build_graph_for(x, cfg, "batched")
    sweep(g0, "r16")
    idx = song.SongIndex(x, g0, metric=cfg.metric)
    t = time.time()
    ids, dists = idx.search(x, params=song.Params(K=2 * D + 1, queue_len=max(a.L, 2 * D + 1)))
    torch.cuda.synchronize()
    res["refine_search_s"] = round(time.time() - t, 2)
    idx.close()
    n = x.shape[0]
    rows = torch.arange(n, device=x.device)[:, None]
    for mode in ("unrestricted", "earlier"):
        keep = (ids != rows) & (ids >= 0)
        if mode == "earlier":
            keep &= ids < rows
        # stable compaction of the kept entries to the front, first D
        order = torch.argsort((~keep).to(torch.int8), dim=1, stable=True)[:, :D]
        fi = torch.gather(ids, 1, order)
        fd = torch.gather(dists, 1, order)
        ok = torch.gather(keep, 1, order)
        fi = torch.where(ok, fi, torch.full_like(fi, -1))
        fd = torch.where(ok, fd, torch.full_like(fd, float("inf")))
        g1 = song.build_graph_from_forward(x, fi, fd, cfg.metric)
        sweep(g1, "refined_" + mode)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
