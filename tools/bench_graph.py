"""Device graph construction (song_build_graph, reading R15) vs the torch
tooling on the SIFT1M-shaped workload: build time (CUDA events) and the
recall@10 of the search at a few queue lengths on each graph.

    python tools/bench_graph.py [--n 1000000]
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
    ap.add_argument("--n", type=int, default=1_000_000)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.graph import build_graph as tool_build
    from workloads.synth import CONFIGS, make_data
    cfg = CONFIGS["sift1m"]
    x, q = make_data(cfg, device="cuda", n=args.n)
    truth = bench.ground_truth(x, q, 10, "l2")
    res = {"workload": f"sift1m-shaped {args.n}x128, degree 32", "builders": {}}
    for name, fn in (("song_build_graph", lambda: song.build_graph(x, 32)),
                     ("torch tooling", lambda: tool_build(x, degree=32))):
        fn() if args.n <= 100_000 else None  # warm-up on small sizes only
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        adj = fn()
        b.record()
        torch.cuda.synchronize()
        sec = a.elapsed_time(b) / 1e3
        idx = song.SongIndex(x, adj)
        curve = []
        for L in (16, 32, 48, 64, 96):
            ids, _ = idx.search(q, params=song.Params(K=10, queue_len=L))
            torch.cuda.synchronize()
            curve.append((L, round(bench.recall_t(ids, truth), 4)))
        idx.close()
        res["builders"][name] = {"seconds": round(sec, 3), "recall_at_10": curve}
        print(f"[graph] {name}: {sec:.2f} s, recall {curve}", file=sys.stderr, flush=True)
    line = json.dumps(res)
    print(line)
    if args.out:
        open(args.out, "w").write(line + "\n")


if __name__ == "__main__":
    main()
