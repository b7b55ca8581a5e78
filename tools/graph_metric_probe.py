"""Which metric should the graph of an inner-product workload be built with?

Builds the GloVe-shaped (IP) index's graph with song_build_graph under each
metric, searches it with the IP metric, and prints recall@10 against the
exact IP top-10 at a few queue lengths.

    python tools/graph_metric_probe.py [--config glove200] [--out gpurun_out/probe.json]
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
    ap.add_argument("--config", default="glove200")
    ap.add_argument("--metrics", default="ip,l2,cosine")
    ap.add_argument("--L", default="32,64,128,256,512,1024")
    ap.add_argument("--out", default="gpurun_out/graph_metric_probe.json")
    a = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS, make_data
    cfg = CONFIGS[a.config]
    x, q = make_data(cfg, device="cuda")
    truth = bench.ground_truth(x, q, cfg.K, cfg.metric)
    res = {"config": cfg.name, "search_metric": cfg.metric}
    for gm in a.metrics.split(","):
        t = time.time()
        if gm.startswith("xbox"):  # MIPS -> L2 reduction: [x, sqrt(M^2 - |x|^2)], L2 graph
            nrm2 = (x * x).sum(1)
            xa = torch.cat([x, (nrm2.max() - nrm2).clamp_min(0).sqrt()[:, None]], 1).contiguous()
            adj = (song.build_graph_batched(xa, cfg.degree, "l2", prefix=1 << 16, queue_len=64)
                   if gm == "xbox-batched" else song.build_graph(xa, cfg.degree, "l2"))
            del xa
        elif gm.endswith("-noheur"):  # torch tooling, plain NSW lists (no heuristic)
            from workloads.graph import build_graph as tool_build
            adj = tool_build(x, cfg.degree, gm[:-len("-noheur")], heuristic=False)
        else:
            adj = song.build_graph(x, cfg.degree, gm)
        torch.cuda.synchronize()
        bt = time.time() - t
        idx = song.SongIndex(x, adj, metric=cfg.metric)
        row = {"build_s": round(bt, 2), "recall": {}}
        for L in map(int, a.L.split(",")):
            ids, _ = idx.search(q, params=song.Params(K=cfg.K, queue_len=L))
            row["recall"][L] = round(bench.recall_t(ids, truth), 4)
        idx.close()
        res[gm] = row
        print(gm, row, flush=True)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
