"""How much of the SIFT1M-shaped step is the persistent grid's tail?

Times the bench's search (L = 48) on the 10,000-query batch and on the same
batch tiled 2x / 4x (more waves amortise the tail), records the per-query
counters, and simulates the ticket scheduler (3552 warp slots, query time
proportional to its expansions + distances) in ticket order and longest-first.

    python tools/tail_sim.py [--L 48] [--out gpurun_out/tail.json]
"""
import argparse
import heapq
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def makespan(cost, slots):
    h = [0.0] * slots
    for c in cost:
        t = heapq.heappop(h)
        heapq.heappush(h, t + c)
    return max(h)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--L", type=int, default=48)
    ap.add_argument("--slots", type=int, default=148 * 24)
    ap.add_argument("--out", default="gpurun_out/tail.json")
    ap.add_argument("--cache", default="")
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS
    cfg = CONFIGS["sift1m"]
    dev = torch.device("cuda", 0)
    x, q0, q, adj = bench.build_workload(cfg, dev, 0, print, a.cache)
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    p = song.Params(K=cfg.K, queue_len=a.L)
    _, _, ctr = idx.search(q, params=p, counters=True)
    ctr = ctr.cpu().numpy().astype(np.float64)
    res = {"L": a.L}
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for rep in (1, 2, 4, 8):
        qq = q.repeat(rep, 1).contiguous()
        out = (torch.empty((qq.shape[0], cfg.K), dtype=torch.int32, device=dev),
               torch.empty((qq.shape[0], cfg.K), dtype=torch.float32, device=dev), None)
        for _ in range(3):
            idx.search(qq, params=p, out=out)
        ts = []
        for _ in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            idx.search(qq, params=p, out=out)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        res[f"x{rep}"] = {"nq": int(qq.shape[0]), "ms": ms, "qps": qq.shape[0] / ms * 1e3}
    # scheduler simulation, cost = expansions (the sequential iterations)
    for name, cost in (("exp", ctr[:, 1]), ("dist", ctr[:, 0]), ("mix", ctr[:, 1] + ctr[:, 0] / 16)):
        ideal = cost.sum() / a.slots
        res[f"sim_{name}"] = {
            "ideal": ideal, "ticket_order": makespan(cost, a.slots) / ideal,
            "longest_first": makespan(np.sort(cost)[::-1], a.slots) / ideal,
            "max_over_mean": float(cost.max() / cost.mean()),
            "p99_over_mean": float(np.percentile(cost, 99) / cost.mean())}
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
