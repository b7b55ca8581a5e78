"""Fig. 10 on B200: where a batched search spends its time.

    python tools/fig10_split.py --config glove200 --queue-lens 50,100,500,1000

Two splits per queue size, on the config's 10,000-query batch (GIST: 1,000
queries x 10):

* end to end (Fig. 10 top, P:1385-1407 / P:1501-1523): HtoD of the query
  batch from pinned memory, the search kernel(s), DtoH of ids + distances —
  each bracketed by CUDA events on one stream, L2 flushed before each run;
* in the kernel (Fig. 10 bottom, P:1443-1465 / P:1559-1581): SM cycles per
  stage from a SONG_STAGE_TIMING build of libsong (built here into
  build_stages/, never the product library): pop / topk update (a3),
  candidate locating (a4), bulk distance (a5), maintenance (a6).  The paper
  counts the queue pop with maintenance; both groupings are printed.

Prints one JSON line; the per-stage shares are of the instrumented kernel
(clock64 reads perturb the schedule slightly; the split, not the absolute
time, is the measurement).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

STAGE_LIB = os.path.join(ROOT, "paper_conf_icde_zhaotl20_b200", "libsong_stages.so")


def build_stage_lib():
    from paper_conf_icde_zhaotl20_b200 import _build
    return _build.build(defines=("SONG_STAGE_TIMING",), out=STAGE_LIB)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="glove200")
    ap.add_argument("--queue-lens", default="50,100,500,1000")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--graph", default="auto")
    ap.add_argument("--out", default="")
    ap.add_argument("--child", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    if not args.child:
        # the instrumented library must be the one the child process maps
        build_stage_lib()
        env = dict(os.environ, SONG_LIB=STAGE_LIB)
        sys.exit(subprocess.call([sys.executable, os.path.abspath(__file__), "--child",
                                  *sys.argv[1:]], env=env))

    import torch
    import bench
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS

    assert song.LIB_PATH == STAGE_LIB, song.LIB_PATH
    log = lambda m: print(f"[fig10] {m}", file=sys.stderr, flush=True)  # noqa: E731
    cfg = CONFIGS[args.config]
    dev = torch.device("cuda", 0)
    x, q0, q, adj = bench.build_workload(cfg, dev, 0, log, "", args.graph)
    truth = bench.ground_truth(x, q0, cfg.K, cfg.metric)
    reps = bench.QUERY_REPLICAS.get(cfg.name, 1)
    qb = q0.repeat(reps, 1).contiguous() if reps > 1 else q0
    idx = song.SongIndex(x, adj, metric=cfg.metric)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    qh = torch.empty(qb.shape, dtype=torch.float32, pin_memory=True)
    qh.copy_(qb.cpu())
    nq = qb.shape[0]
    ih = torch.empty((nq, cfg.K), dtype=torch.int32, pin_memory=True)
    dh = torch.empty((nq, cfg.K), dtype=torch.float32, pin_memory=True)
    qd = torch.empty_like(qb)
    ids = torch.empty((nq, cfg.K), dtype=torch.int32, device=dev)
    dists = torch.empty((nq, cfg.K), dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream(dev)
    rows = []
    for L in [int(v) for v in args.queue_lens.split(",")]:
        if L < cfg.K:
            continue
        p = song.Params(K=cfg.K, queue_len=L)
        r_ids, _ = idx.search(q0, params=p)
        rec = bench.recall_t(r_ids, truth)
        for _ in range(2):
            idx.search(qb, params=p, out=(ids, dists, None))
        torch.cuda.synchronize()
        idx.stage_cycles(reset=True)
        t = {"htod": 0.0, "kernel": 0.0, "dtoh": 0.0}
        for _ in range(args.reps):
            flush.zero_()
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            ev[0].record(stream)
            qd.copy_(qh, non_blocking=True)
            ev[1].record(stream)
            idx.search(qd, params=p, out=(ids, dists, None))
            ev[2].record(stream)
            ih.copy_(ids, non_blocking=True)
            dh.copy_(dists, non_blocking=True)
            ev[3].record(stream)
            torch.cuda.synchronize()
            t["htod"] += ev[0].elapsed_time(ev[1])
            t["kernel"] += ev[1].elapsed_time(ev[2])
            t["dtoh"] += ev[2].elapsed_time(ev[3])
        idx.last_status()
        cyc = [int(c) for c in idx.stage_cycles(reset=True)]
        tot = sum(t.values())
        ctot = max(1, sum(cyc))
        row = {"queue_len": L, f"recall_at_{cfg.K}": round(rec, 4),
               "ms": {k: round(v / args.reps, 4) for k, v in t.items()},
               "share_e2e": {k: round(v / tot, 4) for k, v in t.items()},
               "stage_cycles": dict(zip(["pop_topk", "locate", "distance", "maintain"], cyc)),
               "share_kernel": {"pop_topk": round(cyc[0] / ctot, 4), "locate": round(cyc[1] / ctot, 4),
                                "distance": round(cyc[2] / ctot, 4),
                                "maintain": round(cyc[3] / ctot, 4)},
               "share_kernel_paper_grouping": {
                   "locate": round(cyc[1] / ctot, 4), "distance": round(cyc[2] / ctot, 4),
                   "maintain (incl. pop/topk)": round((cyc[0] + cyc[3]) / ctot, 4)},
               "qps_instrumented": round(nq / (t["kernel"] / args.reps / 1e3), 1)}
        log(json.dumps(row))
        rows.append(row)
    out = {"figure": "Fig. 10 (P:1351-1581) on B200", "config": cfg.name, "nq": nq,
           "graph": bench.default_graph(cfg) if args.graph == "auto" else args.graph,
           "library": "SONG_STAGE_TIMING build (clock64 at stage boundaries, lane 0 of each warp)",
           "rows": rows}
    line = json.dumps(out)
    print(line)
    if args.out:
        with open(args.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
