"""Recall against queue_len for mixed graphs (reading R18's row merge on any
two builders): row = the first `take` links of graph A, then graph B's.

    python tools/mix_graph_probe.py --config sift1m --a batched:l2 --b exact:l2 --take 8,16,24
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def build(spec, x, cfg, song, bq=128, bs=2):
    """spec = kind:metric[:build_queue_len:batch_shift]"""
    parts = spec.split(":")
    kind, metric = parts[0], parts[1]
    if len(parts) == 4:
        bq, bs = int(parts[2]), int(parts[3])
    if kind == "exact":
        return song.build_graph(x, cfg.degree, metric)
    return song.build_graph_batched(x, cfg.degree, metric, prefix=1 << 16, queue_len=bq,
                                    batch_shift=bs)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sift1m")
    ap.add_argument("--a", default="batched:l2")
    ap.add_argument("--b", default="exact:l2")
    ap.add_argument("--take", default="32,24,16,8")
    ap.add_argument("--L", default="16,20,24,28,32,40,48")
    ap.add_argument("--bq", type=int, default=128, help="R16 build queue_len")
    ap.add_argument("--bs", type=int, default=2, help="R16 batch_shift")
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS, make_data
    cfg = CONFIGS[a.config]
    log = lambda m: print(f"[probe] {m}", file=sys.stderr, flush=True)  # noqa: E731
    x, q0 = make_data(cfg, device="cuda")
    truth = bench.ground_truth(x, q0, cfg.K, cfg.metric)
    ga, gb = build(a.a, x, cfg, song, a.bq, a.bs), build(a.b, x, cfg, song, a.bq, a.bs)
    res = {"config": cfg.name, "a": a.a, "b": a.b, "bq": a.bq, "bs": a.bs, "recall": {}, "qps": {}}
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for k in map(int, a.take.split(",")):
        adj = ga if k >= cfg.degree else song.merge_graph_rows(ga, gb, k)
        idx = song.SongIndex(x, adj, metric=cfg.metric)
        row, qrow = {}, {}
        for L in map(int, a.L.split(",")):
            p = song.Params(K=cfg.K, queue_len=L)
            ids, _ = idx.search(q0, params=p)
            row[L] = round(bench.recall_t(ids, truth), 4)
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
            qrow[L] = round(q0.shape[0] / (sum(ms) / len(ms) / 1e3), 1)
        idx.close()
        res["recall"][k], res["qps"][k] = row, qrow
        log(f"take {k}: recall {row} qps {qrow}")
    line = json.dumps(res)
    print(line)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
