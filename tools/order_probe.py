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
    keys = {"ticket": None, "n_exp": ctr[:, 1].float(), "d_entry": ((q - x[0]) ** 2).sum(1),
            "norm": (q * q).sum(1), "d_centroid": ((q - x.mean(0)) ** 2).sum(1)}
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    out = (torch.empty((q.shape[0], cfg.K), dtype=torch.int32, device=dev),
           torch.empty((q.shape[0], cfg.K), dtype=torch.float32, device=dev), None)
    res = {}
    for name, k in keys.items():
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
