"""Fig. 11 on B200: QPS against the query batch size.

    python tools/fig11_batch.py [--batches 100,1000,10000,100000,1000000]

The SIFT1M-shaped index with the bench's graph (R16), batches of fresh
queries from the same generator, top-100 at queue_len 100 (Fig. 11 is the
top-100 experiment) and top-10 at the headline's queue_len; each
point is the CUDA-event time of one batched search (L2 flushed before it),
mean of --reps after warm-up.  Prints one JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batches", default="100,1000,10000,100000,1000000")
    ap.add_argument("--points", default="100:100,10:28", help="K:queue_len pairs")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS, generator_for

    log = lambda m: print(f"[fig11] {m}", file=sys.stderr, flush=True)  # noqa: E731
    cfg = CONFIGS["sift1m"]
    dev = torch.device("cuda", 0)
    x, q0, _, adj = bench.build_workload(cfg, dev, 0, log)
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    gen = generator_for(cfg, dev)
    nmax = max(int(b) for b in args.batches.split(","))
    qall = gen.sample(nmax, cfg.seed + 7)  # fresh queries (never base rows)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    rows = []
    for pt in args.points.split(","):
        K, L = (int(v) for v in pt.split(":"))
        p = song.Params(K=K, queue_len=L)
        for b in [int(v) for v in args.batches.split(",")]:
            q = qall[:b].contiguous()
            out = (torch.empty((b, K), dtype=torch.int32, device=dev),
                   torch.empty((b, K), dtype=torch.float32, device=dev), None)
            for _ in range(2):
                idx.search(q, params=p, out=out)
            ms = []
            for _ in range(args.reps):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                idx.search(q, params=p, out=out)
                e1.record()
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            idx.last_status()
            t = sum(ms) / len(ms)
            row = {"K": K, "queue_len": L, "batch": b, "ms": round(t, 4),
                   "qps": round(b / (t / 1e3), 1)}
            log(json.dumps(row))
            rows.append(row)
    res = {"figure": "Fig. 11 (P:1593-1631) on B200", "workload": f"sift1m-shaped, {bench.GRAPH_DESC[bench.default_graph(cfg)]}",
           "rows": rows}
    line = json.dumps(res)
    print(line)
    if args.out:
        with open(args.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
