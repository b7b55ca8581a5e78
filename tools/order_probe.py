"""Measured effect of the ticket order on the 10,000-query SIFT1M-shaped step:
the same search on the batch permuted by a few keys (descending), CUDA events,
L2 flushed between runs.  'n_exp' (the query's own expansions) is the
longest-first upper bound.

    python tools/order_probe.py [--out gpurun_out/order_probe.json]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--L", type=int, default=48)
    ap.add_argument("--out", default="gpurun_out/order_probe.json")
    ap.add_argument("--cache", default="")
    ap.add_argument("--only", default="")
    ap.add_argument("--schedule", default="batch")
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS
    cfg = CONFIGS["sift1m"]
    dev = torch.device("cuda", 0)
    x, q0, q, adj = bench.build_workload(cfg, dev, 0, print, a.cache)
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    p = song.Params(K=cfg.K, queue_len=a.L, schedule=a.schedule)
    _, _, ctr = idx.search(q, params=p, counters=True)
    keys = {"ticket": None, "n_exp": ctr[:, 1].float(), "d_entry": ((q - x[0]) ** 2).sum(1),
            "norm": (q * q).sum(1), "d_centroid": ((q - x.mean(0)) ** 2).sum(1)}
    g = torch.Generator(device="cuda").manual_seed(5)
    for m in (64, 256, 1024):
        sm = x[torch.randint(0, x.shape[0], (m,), device="cuda", generator=g)]
        d = (q * q).sum(1, keepdim=True) + (sm * sm).sum(1)[None] - 2 * q @ sm.T
        keys[f"mean10_of_{m}"] = d.topk(min(10, m), dim=1, largest=False).values.mean(1)
        keys[f"mean_of_{m}"] = d.mean(1)
    rk = lambda v: torch.argsort(torch.argsort(v)).float()
    keys["rank_centroid+mean10_256"] = rk(keys["d_centroid"]) + rk(keys["mean10_of_256"])
    keys["d_centroid_x_mean10_256"] = keys["d_centroid"] * keys["mean10_of_256"]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    out = (torch.empty((q.shape[0], cfg.K), dtype=torch.int32, device=dev),
           torch.empty((q.shape[0], cfg.K), dtype=torch.float32, device=dev), None)
    res = {}
    for name, k in [(n, keys[n]) for n in (a.only.split(",") if a.only else keys)]:
        qq = q if k is None else q[torch.argsort(k, descending=True)].contiguous()
        for _ in range(3):
            idx.search(qq, params=p, out=out)
        ts = []
        for _ in range(20):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            idx.search(qq, params=p, out=out)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        res[name] = {"ms_median": float(np.median(ts)), "qps": q.shape[0] / float(np.median(ts)) * 1e3}
        print(name, res[name], flush=True)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
