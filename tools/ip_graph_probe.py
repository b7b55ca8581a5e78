"""IP workload: recall@10 against queue_len for mixed graphs — each row takes
its first `a` neighbours from the IP graph and fills the rest from the cosine
(angular) graph (ids de-duplicated), both built by song_build_graph (R15).

    python tools/ip_graph_probe.py --mix 32,24,16 --out gpurun_out/ip_graph_probe.json
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def mix_rows(a_ip, a_cos, k):
    """row = first k of the IP row, then the cosine row's ids not already in it,
    then the rest of the IP row; -1 padded (torch, on the device)."""
    import torch
    n, D = a_ip.shape
    cand = torch.cat([a_ip[:, :k], a_cos, a_ip[:, k:]], 1)  # [n, 2D]
    # drop repeats: keep the first occurrence of each id in the row
    srt, order = torch.sort(cand, dim=1, stable=True)
    dup = torch.zeros_like(cand, dtype=torch.bool)
    dup_s = torch.zeros_like(srt, dtype=torch.bool)
    dup_s[:, 1:] = srt[:, 1:] == srt[:, :-1]
    dup.scatter_(1, order, dup_s)
    cand = torch.where(dup | (cand < 0), torch.full_like(cand, -1), cand)
    # compact the kept ids to the front, preserving order
    key = torch.where(cand >= 0, torch.arange(2 * D, device=cand.device)[None].expand_as(cand),
                      torch.full_like(cand, 10 ** 6))
    idx = torch.argsort(key, dim=1, stable=True)[:, :D]
    return torch.gather(cand, 1, idx).to(torch.int32).contiguous()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="glove200")
    ap.add_argument("--mix", default="32,24,16,8")
    ap.add_argument("--L", default="64,128,256,512,768,1024,1280")
    ap.add_argument("--cos-builder", default="exact", choices=["exact", "batched"])
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS
    cfg = CONFIGS[a.config]
    log = lambda m: print(f"[probe] {m}", file=sys.stderr, flush=True)  # noqa: E731
    x, q0, _, a_ip = bench.build_workload(cfg, torch.device("cuda", 0), 0, log, "/tmp/w_glove200.pt")
    truth = bench.ground_truth(x, q0, cfg.K, cfg.metric)
    if a.cos_builder == "batched":
        b = bench.BUILD
        a_cos = song.build_graph_batched(x, cfg.degree, "cosine", prefix=b["prefix"],
                                         queue_len=b["queue_len"], batch_shift=b["batch_shift"])
    else:
        a_cos = song.build_graph(x, cfg.degree, "cosine")
    res = {"config": cfg.name, "cos_builder": a.cos_builder, "recall": {}}
    for k in map(int, a.mix.split(",")):
        adj = a_ip if k >= cfg.degree else mix_rows(a_ip, a_cos, k)
        idx = song.SongIndex(x, adj, metric=cfg.metric)
        row = {}
        for L in map(int, a.L.split(",")):
            ids, _ = idx.search(q0, params=song.Params(K=cfg.K, queue_len=L))
            row[L] = round(bench.recall_t(ids, truth), 4)
        idx.close()
        res["recall"][f"ip{k}+cos{cfg.degree - k}"] = row
        log(f"ip {k} + cos: {row}")
    line = json.dumps(res)
    print(line)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
