"""Three-graph R18 row merges: recall / QPS against queue_len.
M = merge(merge(A, B, t1), C, t2).

    python tools/mix3_probe.py --config sift1m --a batched:l2:128:2 --b batched:l2:64:1 \\
        --c exact:l2 --takes 16/24,20/28 --L 14,16,18,20
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import bench  # noqa: E402
from mix_graph_probe import build  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sift1m")
    ap.add_argument("--a", default="batched:l2:128:2")
    ap.add_argument("--b", default="batched:l2:64:1")
    ap.add_argument("--c", default="exact:l2")
    ap.add_argument("--takes", default="12/24,16/24,16/28,20/28,10/20")
    ap.add_argument("--L", default="14,16,18,20")
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS, make_data
    cfg = CONFIGS[a.config]
    x, q0 = make_data(cfg, device="cuda")
    truth = bench.ground_truth(x, q0, cfg.K, cfg.metric)
    A, B, C = (build(s, x, cfg, song) for s in (a.a, a.b, a.c))
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    res = {"config": cfg.name, "a": a.a, "b": a.b, "c": a.c, "rows": {}}
    for tt in a.takes.split(","):
        t1, t2 = (int(v) for v in tt.split("/"))
        adj = song.merge_graph_rows(song.merge_graph_rows(A, B, t1), C, t2)
        idx = song.SongIndex(x, adj, metric=cfg.metric)
        row = {}
        for L in map(int, a.L.split(",")):
            p = song.Params(K=10, queue_len=L)
            ids, _ = idx.search(q0, params=p)
            r = bench.recall_t(ids, truth)
            for _ in range(3):
                idx.search(q0, params=p)
            ms = []
            for _ in range(5):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                idx.search(q0, params=p)
                e1.record()
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            row[L] = (round(r, 4), round(q0.shape[0] / (sum(ms) / 5 / 1e3), 1))
        idx.close()
        res["rows"][tt] = row
        print(a.config, tt, row, flush=True)
    line = json.dumps(res)
    print(line)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
