"""IP workload: recall@10 against queue_len for a few entry vertices and graphs
(the search's `entry` parameter; Alg. 1's "default starting point").

    python tools/ip_entry_probe.py --out gpurun_out/ip_entry_probe.json
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
    ap.add_argument("--config", default="glove200")
    ap.add_argument("--L", default="64,128,256,512,768,1024,1280")
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS
    cfg = CONFIGS[a.config]
    log = lambda m: print(f"[probe] {m}", file=sys.stderr, flush=True)  # noqa: E731
    x, q0, _, adj = bench.build_workload(cfg, torch.device("cuda", 0), 0, log, "/tmp/w_glove200.pt")
    truth = bench.ground_truth(x, q0, cfg.K, cfg.metric)
    norms = x.norm(dim=1)
    qm = q0.mean(0)
    entries = {"0": 0, "max_norm": int(norms.argmax()), "max_ip_mean_query": int((x @ qm).argmax()),
               "median_norm": int(norms.argsort()[len(norms) // 2])}
    res = {"config": cfg.name, "graph": bench.default_graph(cfg), "entries": entries, "recall": {}}
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    for name, e in entries.items():
        row = {}
        for L in map(int, a.L.split(",")):
            ids, _ = idx.search(q0, params=song.Params(K=cfg.K, queue_len=L, entry=e))
            row[L] = round(bench.recall_t(ids, truth), 4)
        res["recall"][name] = row
        log(f"{name} (id {e}): {row}")
    line = json.dumps(res)
    print(line)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
