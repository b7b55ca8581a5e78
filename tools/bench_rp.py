"""Fig. 14 on B200 (§VII): QPS-recall curves of the search over
1-bit random-projection codes vs over the original vectors, MNIST1m-shaped.

    python tools/bench_rp.py [--n 1000000] [--bits 128,256,512] [--steps 5]

Pipeline (all through the C ABI): MNIST-shaped integer images [n, 784] built
on the device; the degree-32 graph built on the ORIGINAL vectors;
``song_index_create_rp`` streams the vectors from host memory through the
encoder and keeps only the codes ("the hashed dataset may fit in GPU
memory"); queries are encoded by the same R inside ``song_search_ex``.
Recall@1 ("top-1", Fig. 14) is against the exact nearest neighbour of the
ORIGINAL vectors (reading R12).  Each point: CUDA-event time of the search
(encode + search kernels for the hashed arm), L2 flushed between steps.
Prints one JSON line (supplementary: the driver's bench line is bench.py's).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402  (helpers only: ground truth, recall, clocks, peaks)

GRID = [1, 2, 4, 8, 12, 16, 24, 32, 48, 64, 96, 128, 192, 256, 384, 512]


def hamming_min(codes, qcodes):
    """Exact minimum Hamming distance of every query code over all codes (torch
    SWAR popcount on int64 lanes; ground truth for the search over codes)."""
    import torch
    m = 0xffffffff
    c = codes.long() & m
    out = []
    for s in range(0, qcodes.shape[0], 16):
        q = qcodes[s:s + 16].long() & m
        x = q[:, None, :] ^ c[None]                       # [16, n, W]
        x = x - ((x >> 1) & 0x55555555)
        x = (x & 0x33333333) + ((x >> 2) & 0x33333333)
        x = (((x + (x >> 4)) & 0x0F0F0F0F) * 0x01010101 & m) >> 24
        out.append(x.sum(2).min(1).values)
    return torch.cat(out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1_000_000)
    ap.add_argument("--nq", type=int, default=10_000)
    ap.add_argument("--bits", default="64,128,256,512")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--max-L", type=int, default=512)
    ap.add_argument("--config", default="mnist1m", choices=["mnist1m", "mnist8m"])
    ap.add_argument("--builder", default="exact", choices=["exact", "batched"],
                    help="graph on the original vectors: exact insertion (workloads.graph, "
                         "O(n^2)) or the library's batched-insertion builder (R16; MNIST8m)")
    ap.add_argument("--out", default="")
    args = ap.parse_args()

    import numpy as np
    import torch
    from paper_conf_icde_zhaotl20_b200 import song
    from workloads.graph import build_graph
    from workloads.synth import CONFIGS, MnistLike, rp_matrix

    log = lambda m: print(f"[bench_rp] {m}", file=sys.stderr, flush=True)  # noqa: E731
    cfg = CONFIGS[args.config]
    dev = torch.device("cuda", 0)
    t0 = time.time()
    gen = MnistLike(cfg.dim, cfg.seed, dev)
    x = gen.sample(args.n, cfg.seed)
    q = gen.sample(args.nq, cfg.seed + 1)
    if args.builder == "batched":
        b = bench.BUILD
        adj = song.build_graph_batched(x, cfg.degree, "l2", prefix=b["prefix"],
                                       queue_len=b["queue_len"], batch_shift=b["batch_shift"])
    else:
        adj = build_graph(x, degree=cfg.degree, metric="l2")
    torch.cuda.synchronize()
    log(f"data + graph {time.time() - t0:.1f}s")
    truth = bench.ground_truth(x, q, 1, "l2")
    torch.cuda.empty_cache()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def curve(idx, label, bytes_per_dist, ham_truth=None):
        pts = []
        for L in GRID:
            if L > args.max_L:
                break
            p = song.Params(K=1, queue_len=L)
            ids, dd, ctr = idx.search(q, params=p, counters=True)
            torch.cuda.synchronize()
            idx.last_status()
            rec = bench.recall_t(ids, truth)
            # search quality in code space: found distance == exact min Hamming distance
            rec_h = (None if ham_truth is None else
                     round(float((dd[:, 0].long() <= ham_truth).float().mean()), 4))
            n_dist = int(ctr[:, 0].long().sum())
            n_exp = int(ctr[:, 1].long().sum())
            for _ in range(args.warmup):
                idx.search(q, params=p)
            ms = []
            for _ in range(args.steps):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                idx.search(q, params=p)
                b.record()
                torch.cuda.synchronize()
                ms.append(a.elapsed_time(b))
            t = sum(ms) / len(ms) / 1e3
            alg = bytes_per_dist * n_dist + 4 * cfg.degree * n_exp
            pts.append({"L": L, "recall_at_1": round(rec, 4), "recall_hamming_at_1": rec_h,
                        "qps": round(args.nq / t, 1),
                        "ms": round(t * 1e3, 4), "n_dist_per_q": round(n_dist / args.nq, 1),
                        "alg_GBps": round(alg / t / 1e9, 1)})
            log(f"{label} L={L} recall@1={rec:.4f} (code space {rec_h}) qps={args.nq / t:,.0f}")
            if rec >= 0.999 or (rec_h is not None and rec_h >= 0.999):
                break
        return pts

    result = {"figure": "Fig. 14 (P:1823) / Table IV (P:1827-1831) on B200", "workload":
              f"{cfg.name}-shaped: {args.n}x784 integer pixels, L2, degree-32 graph "
              f"({args.builder} builder) on the original vectors, {args.nq} queries, top-1",
              "curves": {}, "encode": {}}
    # original vectors ("SONG" line of Fig. 14)
    idx = song.SongIndex(x, adj, metric="l2")
    result["curves"]["original-784"] = curve(idx, "original", 4 * 784)
    idx.close()
    xh = x.cpu().numpy()
    adjh = adj.cpu().numpy()
    del x
    torch.cuda.empty_cache()
    for bits in [int(b) for b in args.bits.split(",")]:
        R = rp_matrix(bits, 784, cfg.seed + 3).numpy()
        torch.cuda.synchronize()
        t = time.perf_counter()
        idx = song.SongIndex.from_rp(xh, R, adjh)  # host vectors streamed, codes kept
        torch.cuda.synchronize()
        enc_s = time.perf_counter() - t
        info = idx.info()
        result["encode"][f"hash-{bits}"] = {
            "create_rp_s": round(enc_s, 3), "code_bytes": info.vector_bytes,
            "original_bytes": args.n * 784 * 4,
            "reduction": round(args.n * 784 * 4 / info.vector_bytes, 1)}
        log(f"hash-{bits}: create_rp {enc_s:.2f}s, codes {info.vector_bytes / 2**20:.1f} MiB")
        Rt = torch.as_tensor(R, device=dev)
        ham_truth = hamming_min(song.rp_encode(torch.as_tensor(xh, device=dev), Rt),
                                song.rp_encode(q, Rt))
        result["curves"][f"hash-{bits}"] = curve(idx, f"hash-{bits}", bits // 8, ham_truth)
        idx.close()
    result["clocks_note"] = "device-timed with CUDA events; L2 flushed between steps"
    line = json.dumps(result)
    print(line)
    if args.out:
        with open(args.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
