"""Fig. 9 on B200 (§V): QPS-recall@10 of multi-step probing
(steps = 1, 2, 4 pops per iteration) on the SIFT1M-shaped workload, plus the
visited-set variants of Fig. 7 at the same operating points.

    python tools/bench_knobs.py [--steps-list 1,2,4] [--visited hash,bloom]

Each point: one batched search of the 10,000 queries, CUDA-event timed over
--reps runs after warm-up, L2 flushed between runs.  Prints one JSON line
(supplementary to bench.py's line).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402

GRID = [10, 16, 24, 32, 48, 64, 96, 128, 192, 256]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sift1m")
    ap.add_argument("--steps-list", default="1,2,4")
    ap.add_argument("--visited", default="hash,bloom,hashtable,hashtable-sel,cuckoo")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--cache", default="")
    ap.add_argument("--out", default="")
    args = ap.parse_args()

    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS

    log = lambda m: print(f"[knobs] {m}", file=sys.stderr, flush=True)  # noqa: E731
    cfg = CONFIGS[args.config]
    dev = torch.device("cuda", 0)
    x, q0, q, adj = bench.build_workload(cfg, dev, 0, log, args.cache)
    truth = bench.ground_truth(x, q0, cfg.K, cfg.metric)
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def point(p):
        ids, _, ctr = idx.search(q0, params=p, counters=True)
        torch.cuda.synchronize()
        idx.last_status()
        rec = bench.recall_t(ids, truth)
        for _ in range(3):
            idx.search(q0, params=p)
        ms = []
        for _ in range(args.reps):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            idx.search(q0, params=p)
            b.record()
            torch.cuda.synchronize()
            ms.append(a.elapsed_time(b))
        t = sum(ms) / len(ms) / 1e3
        nq = q0.shape[0]
        return {"recall_at_10": round(rec, 4), "qps": round(nq / t, 1), "ms": round(t * 1e3, 4),
                "n_dist_per_q": round(float(ctr[:, 0].float().mean()), 1),
                "n_exp_per_q": round(float(ctr[:, 1].float().mean()), 1)}

    res = {"figure": "Fig. 9 / Fig. 7 on B200", "workload":
           f"{cfg.name}-shaped {cfg.n}x{cfg.dim} {cfg.metric}, degree {cfg.degree}, "
           f"{q0.shape[0]} queries, K={cfg.K}", "multi_step": {}, "visited": {}}
    for st in [int(v) for v in args.steps_list.split(",")]:
        pts = []
        for L in GRID:
            r = point(song.Params(K=cfg.K, queue_len=L, steps=st))
            r["L"] = L
            pts.append(r)
            log(f"steps={st} L={L} {r}")
        res["multi_step"][f"steps={st}"] = pts
    for vk in args.visited.split(","):
        pts = []
        for L in GRID:
            r = point(song.Params(K=cfg.K, queue_len=L, visited=vk))
            r["L"] = L
            pts.append(r)
            log(f"visited={vk} L={L} {r}")
        res["visited"][vk] = pts
    idx.close()
    line = json.dumps(res)
    print(line)
    if args.out:
        with open(args.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
