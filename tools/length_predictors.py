"""Is there a cheap a-priori predictor of a query's search length?

For the SIFT1M-shaped batch at L = 48: per-query expansions (the counters)
against cheap features, Spearman rank correlation, and the simulated
persistent-grid makespan (3552 warp slots) when tickets are issued in the
order of each feature (descending) vs ticket order.

    python tools/length_predictors.py [--out gpurun_out/predictors.json]
"""
import argparse
import heapq
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def makespan(cost, slots):
    h = [0.0] * slots
    for c in cost:
        heapq.heappush(h, heapq.heappop(h) + c)
    return max(h)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--L", type=int, default=48)
    ap.add_argument("--slots", type=int, default=148 * 24)
    ap.add_argument("--out", default="gpurun_out/predictors.json")
    ap.add_argument("--cache", default="")
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS
    cfg = CONFIGS["sift1m"]
    x, q0, q, adj = bench.build_workload(cfg, torch.device("cuda", 0), 0, print, a.cache)
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    _, _, ctr = idx.search(q, params=song.Params(K=cfg.K, queue_len=a.L), counters=True)
    exp = ctr[:, 1].double().cpu().numpy()
    feats = {}
    feats["d_entry"] = ((q - x[0]) ** 2).sum(1)
    feats["norm"] = (q * q).sum(1)
    g = torch.Generator(device="cuda").manual_seed(5)
    for m in (256, 4096):
        sm = x[torch.randint(0, x.shape[0], (m,), device="cuda", generator=g)]
        d = (q * q).sum(1, keepdim=True) + (sm * sm).sum(1)[None] - 2 * q @ sm.T
        feats[f"nn_of_{m}"] = d.min(1).values
        feats[f"mean10_of_{m}"] = d.topk(10, dim=1, largest=False).values.mean(1)
    _, _, c1 = idx.search(q, params=song.Params(K=1, queue_len=1), counters=True)
    feats["greedy_hops"] = c1[:, 1].float()
    _, _, c8 = idx.search(q, params=song.Params(K=8, queue_len=8), counters=True)
    feats["exp_L8"] = c8[:, 1].float()
    from scipy.stats import spearmanr
    ideal = exp.sum() / a.slots
    res = {"L": a.L, "mean_exp": float(exp.mean()), "ticket_order": makespan(exp, a.slots) / ideal,
           "oracle_lpt": makespan(np.sort(exp)[::-1], a.slots) / ideal, "features": {}}
    for k, v in feats.items():
        v = v.double().cpu().numpy()
        rho = float(spearmanr(v, exp).correlation)
        order = np.argsort(-v if rho > 0 else v, kind="stable")
        res["features"][k] = {"spearman": round(rho, 3),
                              "makespan_sorted": round(makespan(exp[order], a.slots) / ideal, 3)}
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
