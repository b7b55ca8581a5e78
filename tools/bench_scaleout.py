"""Scale-out config (BASELINE.json configs[4]) on one B200: the SIFT-shaped
generator at n rows (default 100M), the graph built by song_build_graph_batched
(reading R16: the exact R15 builder is O(n^2)), then QPS at
recall@10 >= 0.95 over 10,000 fresh queries (query-sharded mode: every GPU of
the scale-out holds this replica and searches its own batch).  With
--compare-exact (n <= a few million) the R15 graph is built too and both
recall curves are reported.

    python tools/bench_scaleout.py [--n 100000000] [--out gpurun_out/scaleout.json]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

GRID = [10, 12, 16, 20, 24, 32, 40, 48, 64, 80, 96, 128, 160, 192, 256]


def exact_topk(x, q, K, qchunk=1024, xchunk=1 << 21):
    """Brute-force top-K (squared L2, fp32 GEMM, TF32 off; exact on the integer
    data) over x in chunks, merged by (dist, id)."""
    import torch
    torch.backends.cuda.matmul.allow_tf32 = False
    out = []
    for s in range(0, q.shape[0], qchunk):
        qq = q[s:s + qchunk]
        qn = (qq * qq).sum(1, keepdim=True)
        best_d = torch.full((qq.shape[0], K), float("inf"), device=q.device)
        best_i = torch.full((qq.shape[0], K), -1, dtype=torch.int64, device=q.device)
        for c in range(0, x.shape[0], xchunk):
            xc = x[c:c + xchunk]
            d = qn + (xc * xc).sum(1)[None] - 2 * qq @ xc.T
            v, i = torch.topk(d, K, dim=1, largest=False)
            cd = torch.cat([best_d, v], 1)
            ci = torch.cat([best_i, i + c], 1)
            # (dist, id) order: ids break ties
            key = cd.double() * 4e9 + ci.double()
            o = torch.argsort(key, dim=1)[:, :K]
            best_d, best_i = torch.gather(cd, 1, o), torch.gather(ci, 1, o)
            del d
        out.append(best_i)
    return torch.cat(out).int()


def sharded(a, x, q, truth, song, bench, torch, np):
    """Dataset sharding on one GPU: shard g = rows [lo_g, hi_g) with its own
    R16 graph; each shard searches the whole batch (id_offset = lo_g) — on a
    G-GPU node the G searches run concurrently, so the step is the slowest
    shard's search + the merge — and song_merge_topk keeps the K best."""
    from paper_conf_icde_zhaotl20_b200.sharded import shard_ranges
    G, dev = a.shards, q.device
    idxs = []
    t0 = time.time()
    for lo, hi in shard_ranges(a.n, G):
        adj = song.build_graph_batched(x[lo:hi], 32, "l2", prefix=a.prefix,
                                       queue_len=a.build_queue_len, batch_shift=a.batch_shift)
        idxs.append((lo, song.SongIndex(x[lo:hi], adj)))
        del adj
        torch.cuda.empty_cache()
    build_s = time.time() - t0
    out = {"shards": G, "build_s_total": round(build_s, 1), "sweep": []}
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for L in GRID:
        ids_g, d_g, shard_ms = [], [], []
        for lo, idx in idxs:
            p = song.Params(K=10, queue_len=L, id_offset=lo)
            idx.search(q, params=p)
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            i, d = idx.search(q, params=p)
            e1.record()
            torch.cuda.synchronize()
            shard_ms.append(e0.elapsed_time(e1))
            ids_g.append(i)
            d_g.append(d)
        # the fused gather + merge kernel of the multi-GPU path (song_merge_topk_peers),
        # here reading the G shards' result buffers through a pointer table
        ptr = lambda ts: torch.tensor([t.data_ptr() for t in ts], dtype=torch.int64, device=dev)  # noqa: E731
        pi, pd = ptr(ids_g), ptr(d_g)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        mi, _ = song.merge_topk_peers(pi, pd, q.shape[0], 10, 10)
        e1.record()
        torch.cuda.synchronize()
        mi2, _ = song.merge_topk(torch.stack(ids_g), torch.stack(d_g), 10)
        assert torch.equal(mi, mi2)
        r = bench.recall_t(mi, torch.as_tensor(truth, device=dev))
        step_ms = max(shard_ms) + e0.elapsed_time(e1)
        out["sweep"].append({"L": L, "recall": round(r, 4), "max_shard_ms": round(max(shard_ms), 4),
                             "merge_ms": round(e0.elapsed_time(e1), 4),
                             "qps_G_gpus": round(a.nq / step_ms * 1e3, 1)})
        if r >= 0.95:
            out["queue_len"] = L
            break
    for _, idx in idxs:
        idx.close()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=100_000_000)
    ap.add_argument("--nq", type=int, default=10_000)
    ap.add_argument("--prefix", type=int, default=1 << 16)
    ap.add_argument("--build-queue-len", type=int, default=128)
    ap.add_argument("--batch-shift", type=int, default=2)
    ap.add_argument("--compare-exact", action="store_true")
    ap.add_argument("--mix", default="",
                    help="reading R18 at scale: 'queue_len:shift:take' builds a second R16 graph "
                         "with those builder parameters and searches the row merge (the first "
                         "`take` links of the first graph, then the second's)")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--parity-sample", type=int, default=0,
                    help="queries the oracle recomputes one by one at the operating point")
    ap.add_argument("--shards", type=int, default=0,
                    help="also run dataset sharding (P:471, SURVEY §8(e)(ii)): G shards with "
                         "their own graphs, every query searched on every shard, merged by "
                         "song_merge_topk_peers; emulated on this GPU one shard at a time")
    ap.add_argument("--out", default="gpurun_out/scaleout.json")
    a = ap.parse_args()
    import numpy as np
    import torch
    import bench
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.synth import CONFIGS, generator_for
    cfg = CONFIGS["scaleout100m"]
    dev = torch.device("cuda", 0)
    t0 = time.time()
    gen = generator_for(cfg, dev)
    x = gen.sample(a.n, cfg.seed)
    q = gen.sample(a.nq, cfg.seed + 1)
    torch.cuda.synchronize()
    import psutil
    need = a.n * (128 * 4 + 32 * 4) * 1.6
    if a.parity_sample and psutil.virtual_memory().available < need:
        print(f"parity sample skipped: {psutil.virtual_memory().available / 2**30:.0f} GB host RAM "
              f"available, {need / 2**30:.0f} GB needed", flush=True)
        a.parity_sample = 0
    res = {"host_ram_gb": round(psutil.virtual_memory().total / 2**30, 1), "n": a.n, "nq": a.nq, "dim": 128, "degree": 32, "data_s": round(time.time() - t0, 1),
           "builder": {"prefix": a.prefix, "queue_len": a.build_queue_len,
                       "batch_shift": a.batch_shift}}
    print(res, flush=True)
    t0 = time.time()
    truth = exact_topk(x, q, 10).cpu().numpy()
    torch.cuda.synchronize()
    res["truth_s"] = round(time.time() - t0, 1)
    torch.cuda.empty_cache()
    graphs = {}
    t0 = time.time()
    graphs["batched"] = song.build_graph_batched(x, 32, "l2", prefix=a.prefix,
                                                 queue_len=a.build_queue_len,
                                                 batch_shift=a.batch_shift)
    torch.cuda.synchronize()
    res["build_s"] = round(time.time() - t0, 1)
    print("built", res["build_s"], "s", flush=True)
    if a.mix:
        bq, bs, take = (int(v) for v in a.mix.split(":"))
        t0 = time.time()
        g2 = song.build_graph_batched(x, 32, "l2", prefix=a.prefix, queue_len=bq, batch_shift=bs)
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        graphs["mixed"] = song.merge_graph_rows(graphs["batched"], g2, take)
        del g2
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        res["build_mixed_s"] = round(time.time() - t0, 1)
        res["mix"] = {"second_queue_len": bq, "second_batch_shift": bs, "take": take}
        print("mixed built", res["build_mixed_s"], "s", flush=True)
    if a.compare_exact:
        t0 = time.time()
        graphs["exact"] = song.build_graph(x, 32, "l2")
        torch.cuda.synchronize()
        res["build_exact_s"] = round(time.time() - t0, 1)
    for name, adj in graphs.items():
        idx = song.SongIndex(x, adj)
        adj_host = adj.cpu().numpy() if a.parity_sample else None
        del adj
        graphs[name] = None
        torch.cuda.empty_cache()
        sweep, L_op = [], None
        for L in GRID:
            ids, _ = idx.search(q, params=song.Params(K=10, queue_len=L))
            r = bench.recall_t(ids, torch.as_tensor(truth, device=dev))
            sweep.append((L, round(r, 4)))
            if r >= 0.95 and L_op is None:
                L_op = L
                break
        row = {"recall_sweep": sweep, "queue_len": L_op}
        if L_op:
            p = song.Params(K=10, queue_len=L_op)
            out = (torch.empty((a.nq, 10), dtype=torch.int32, device=dev),
                   torch.empty((a.nq, 10), dtype=torch.float32, device=dev), None)
            _, _, ctr = idx.search(q, params=p, counters=True)
            flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
            for _ in range(3):
                idx.search(q, params=p, out=out)
            ts = []
            for _ in range(a.steps):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                idx.search(q, params=p, out=out)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = float(np.mean(ts))
            if a.parity_sample:
                import oracle
                pick = np.arange(0, a.nq, max(1, a.nq // a.parity_sample))[:a.parity_sample]
                gi, gd, gc = (t.cpu().numpy() for t in idx.search(q, params=p, counters=True))
                t1 = time.time()
                oi, od, oc, _ = oracle.search(x.cpu().numpy(), adj_host, q.cpu().numpy()[pick], 10,
                                              L_op, nthreads=os.cpu_count() or 8,
                                              **bench.oracle_mode(L_op, int(idx.plan(p).visited_cap),
                                                                  queue_kind=int(idx.plan(p).queue_kind)))
                row["parity_sample"] = {
                    "queries": len(pick), "oracle_s": round(time.time() - t1, 1),
                    "ids_equal": float((gi[pick] == oi).all(1).mean()),
                    "dists_equal": float((gd[pick] == od).all(1).mean()),
                    "counters_equal": float((gc[pick].astype(np.int64) == oc).all(1).mean())}
            n_dist, n_exp = int(ctr[:, 0].long().sum()), int(ctr[:, 1].long().sum())
            alg = 512 * n_dist + 128 * n_exp + 512 * a.nq + 80 * a.nq
            peak, _ = bench.measured_peak_hbm()
            row.update({"qps": round(a.nq / ms * 1e3, 1), "ms_per_step": round(ms, 4),
                        "n_dist": n_dist, "n_exp": n_exp,
                        "roofline_frac": round(alg / (ms / 1e3) / 1e9 / peak, 4)})
        idx.close()
        res[name] = row
        print(name, row, flush=True)
    if a.shards:
        res["dataset_sharded"] = sharded(a, x, q, truth, song, bench, torch, np)
        print("dataset_sharded", res["dataset_sharded"], flush=True)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
